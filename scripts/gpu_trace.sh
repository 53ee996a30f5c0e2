for mb in 2 3; do
echo "=== MINB $mb"
GDROID_NVCC_FLAGS="-DGD_MINB=$mb" python -c "import __graft_entry__ as g; g.build()" || exit 1
for w in chain median corpus8 small; do timeout 300 python scripts/trace_rounds.py $w 2>&1 | head -1; done
GDROID_NVCC_FLAGS="-DGD_PHASES -DGD_MINB=$mb" python -c "import __graft_entry__ as g; g.build()" || exit 1
for w in median corpus8; do timeout 300 python scripts/trace_rounds.py $w 2>&1| head -1; done
done
python -c "import __graft_entry__ as g; g.build()"
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
