python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -2
for w in tiny rand small; do timeout 300 python scripts/plain_debug.py $w 2>&1 | tail -4; done
timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -5
WORKLOADS="small median corpus" bash scripts/gpu_ab.sh ""
