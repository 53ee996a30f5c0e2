#!/bin/bash
# Device layout (layout.cu): layout tests, the GPU suite, load timing device vs host layout.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/dl_build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_layout.py -x -q > gpurun_out/dl_layout_tests.log 2>&1
echo "layout tests rc=$?" >> gpurun_out/dl_layout_tests.log
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/dl_gpu_tests.log 2>&1
echo "gpu tests rc=$?" >> gpurun_out/dl_gpu_tests.log
GDROID_TIMING=1 timeout 600 python scripts/load_timing.py 60 > gpurun_out/dl_load_dev.log 2>&1
GDROID_HOST_LAYOUT=1 GDROID_TIMING=1 timeout 600 python scripts/load_timing.py 60 > gpurun_out/dl_load_host.log 2>&1
