#!/bin/bash
# ncu --set full of the heavy-round instantiation on a 16M-node narrow corpus batch, with source
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/nh_build.log 2>&1
timeout 600 python scripts/heavy_batch.py > gpurun_out/nh_plain.log 2>&1
BUILDS=1 timeout 1500 ncu --set full --clock-control none --import-source on --kernel-name-base demangled \
  -k "regex:k_fixpoint.*\(int\)4>" -c 1 -o gpurun_out/nh_heavy python scripts/heavy_batch.py > gpurun_out/nh_ncu.log 2>&1
ncu -i gpurun_out/nh_heavy.ncu-rep --page source --csv --print-source cuda,sass > gpurun_out/nh_source.csv 2>/dev/null
ncu -i gpurun_out/nh_heavy.ncu-rep --page raw --csv > gpurun_out/nh_raw.csv 2>/dev/null
rm -f gpurun_out/nh_heavy.ncu-rep
