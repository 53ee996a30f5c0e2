#!/bin/bash
# Device layout: layout tests, load timing (device vs host layout), default bench.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/dl2_build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_layout.py -x -q > gpurun_out/dl2_layout_tests.log 2>&1
GDROID_TIMING=1 timeout 600 python scripts/load_timing.py 60 > gpurun_out/dl2_load_dev.log 2>&1
timeout 1500 python bench.py > gpurun_out/dl2_bench.jsonl 2> gpurun_out/dl2_bench.err
