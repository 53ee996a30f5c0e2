#!/bin/bash
# ncu --set full (with source) of the worst preset's first k_fixpoint launch at HEAD
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/nw_build.log 2>&1
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:k_fixpoint -c 1 -o gpurun_out/nw_worst \
  python bench.py --workload worst --steps 1 --warmup 0 --no-cpu-baseline --e2e-steps 0 --no-per-config > gpurun_out/nw_ncu.log 2>&1
ncu -i gpurun_out/nw_worst.ncu-rep --page source --csv --print-source cuda,sass > gpurun_out/nw_source.csv 2>/dev/null
ncu -i gpurun_out/nw_worst.ncu-rep --page raw --csv > gpurun_out/nw_raw.csv 2>/dev/null
rm -f gpurun_out/nw_worst.ncu-rep
