#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/fc2_build.log 2>&1
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/fc2_gpu_tests.log 2>&1
GDROID_TIMING=1 timeout 1200 python scripts/e2e_timeline.py 1000 > gpurun_out/fc2_timeline.jsonl 2> gpurun_out/fc2_timeline.err
GDROID_TIMING=1 timeout 600 python scripts/load_timing.py 60 > gpurun_out/fc2_load_dev.log 2>&1
timeout 1500 python bench.py --no-per-config --no-cpu-baseline > gpurun_out/fc2_bench.jsonl 2> gpurun_out/fc2_bench.err
