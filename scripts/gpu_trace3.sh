python -c "import __graft_entry__ as g; g.build()" || exit 1
WORKLOADS="worst" bash scripts/gpu_variants.sh ""
for w in chain small median corpus8; do timeout 300 python scripts/trace_rounds.py $w 2>&1 | tail -9; done
nproc; lscpu | grep "Model name"
