python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -1
timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -4
WORKLOADS="small median corpus worst" bash scripts/gpu_ab.sh "" "-DGD_SMASK=0" "-DGD_PF=1" "-DGD_THREADS=128 -DGD_MINB=7" "-DGD_MINB=4" 2>&1 | grep -v "warning\|Remark\|^ *\^\|^ *$\|uint32_t size\|constexpr int WROWS"
python -c "import paper_conf_ipps_yuwobby20_b200._build as b; b.build(force=True)"
timeout 1500 python scripts/ablation.py --apps 24 --reps 3 --out gpurun_out/ablation_r01.json 2>&1 | tail -34
