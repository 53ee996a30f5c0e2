#!/bin/bash
# Last bench at the final HEAD with the driver's commands.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/f7_smoke.log 2>&1
timeout 2400 python bench.py --gpus 1 --steps 20 --warmup 5 > gpurun_out/f7_bench.jsonl 2> gpurun_out/f7_bench.err; echo "bench rc=$?"
timeout 1800 python bench.py --impl reference --gpus 1 --steps 20 --warmup 5 >> gpurun_out/f7_bench.jsonl 2>> gpurun_out/f7_bench.err; echo "ref rc=$?"
