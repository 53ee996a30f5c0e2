#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/fc_build.log 2>&1
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/fc_gpu_tests.log 2>&1
GDROID_TIMING=1 timeout 1200 python scripts/e2e_timeline.py 1000 > gpurun_out/fc_timeline.jsonl 2> gpurun_out/fc_timeline.err
bash scripts/gpu_ncu_heavy.sh
