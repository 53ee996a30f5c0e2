python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -1
timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -4
WORKLOADS="small median corpus worst" bash scripts/gpu_ab.sh "" "-DGD_MINB=2" 2>&1 | grep -v "warning\|Remark\|^ *\^\|^ *$\|uint32_t size\|constexpr int WROWS"
