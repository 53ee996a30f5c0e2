#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/e2e_build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_layout.py tests/test_gpu_corpus.py -x -q > gpurun_out/e2e_tests.log 2>&1
GDROID_TIMING=1 timeout 1200 python scripts/e2e_timeline.py 1000 > gpurun_out/e2e_timeline3.jsonl 2> gpurun_out/e2e_timeline3.err
timeout 1500 python bench.py --no-per-config > gpurun_out/e2e_bench3.jsonl 2> gpurun_out/e2e_bench3.err
