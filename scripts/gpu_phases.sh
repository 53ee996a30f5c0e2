GDROID_NVCC_FLAGS="-DGD_PHASES" python -c "import __graft_entry__ as g; g.build()" || exit 1
for w in chain median corpus8; do timeout 300 python scripts/trace_rounds.py $w | head -2; done
python -c "import __graft_entry__ as g; g.build()"
