# round protocol + dynamic items + variants: parity, A/B, traces
python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -2
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
WORKLOADS="small median corpus worst" bash scripts/gpu_variants.sh "-DGD_DYN=1" "-DGD_DYN=0"
python -c "import paper_conf_ipps_yuwobby20_b200._build as b; b.build(force=True)"
for w in chain small median corpus8; do timeout 300 python scripts/trace_rounds.py $w 2>&1 | tail -9; done
