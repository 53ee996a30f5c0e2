#!/bin/bash
# Final check at HEAD with the driver's own commands: smoke, GPU suite, bench (--steps 20
# --warmup 5) and the reference arm.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/f4_smoke.log 2>&1; tail -1 gpurun_out/f4_smoke.log
( time timeout 3000 python -m pytest tests -m gpu -q ) > gpurun_out/f4_gpu_tests.log 2>&1; tail -4 gpurun_out/f4_gpu_tests.log
( time timeout 2400 python bench.py --gpus 1 --steps 20 --warmup 5 ) > gpurun_out/f4_bench.jsonl 2> gpurun_out/f4_bench.err; echo "bench rc=$?"
( time timeout 1800 python bench.py --impl reference --gpus 1 --steps 20 --warmup 5 ) >> gpurun_out/f4_bench.jsonl 2>> gpurun_out/f4_bench.err; echo "ref rc=$?"
tail -3 gpurun_out/f4_bench.err
