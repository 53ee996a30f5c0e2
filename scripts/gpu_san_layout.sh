#!/bin/bash
# compute-sanitizer memcheck / racecheck of the device layout kernels on valid and invalid inputs
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/san_build.log 2>&1
CS=/usr/local/cuda/bin/compute-sanitizer
timeout 1500 $CS --tool memcheck --print-limit 50 python scripts/sanitize_layout.py > gpurun_out/san_layout_memcheck.log 2>&1; echo "memcheck rc=$?" >> gpurun_out/san_layout_memcheck.log
timeout 1500 $CS --tool racecheck --print-limit 50 python scripts/sanitize_layout.py > gpurun_out/san_layout_racecheck.log 2>&1; echo "racecheck rc=$?" >> gpurun_out/san_layout_racecheck.log
timeout 1500 $CS --tool memcheck --print-limit 50 python scripts/sanitize_driver.py all > gpurun_out/san_driver_memcheck.log 2>&1; echo "memcheck rc=$?" >> gpurun_out/san_driver_memcheck.log
