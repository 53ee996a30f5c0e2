# dense continuation: parity + A/B of continuation variants
python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -2
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
WORKLOADS="small median corpus worst" bash scripts/gpu_variants.sh "-DGD_CONT_LOAD=4" "-DGD_CONT_LOAD=2" "-DGD_CONT_LOAD=8" "-DGD_CONT_LOAD=4 -DGD_CONT_DEPTH=16" "-DGD_CONT_LOAD=2 -DGD_CONT_DEPTH=32" "-DGD_CONT_LOAD=1 -DGD_CONT_DEPTH=32"
