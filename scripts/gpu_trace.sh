for mb in 3 4 5; do
echo "=== MINB $mb"
GDROID_NVCC_FLAGS="-DGD_MINB=$mb" python -c "import __graft_entry__ as g; g.build()" || exit 1
for w in median corpus8; do timeout 600 python scripts/trace_rounds.py $w 2>&1 | head -1; done
done
python -c "import __graft_entry__ as g; g.build()"
