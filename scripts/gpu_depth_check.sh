#!/bin/bash
# Narrow continuation depth 4 (GD_CONT_DEPTH_NARROW) at HEAD: GPU suite + presets + corpus.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/dc_smoke.log 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/dc_gpu_tests.log 2>&1
out=gpurun_out/dc_bench.log
: > $out
for w in small median worst; do
  echo "== $w" >> $out
  timeout 600 python bench.py --workload $w --steps 10 --warmup 3 --no-cpu-baseline --e2e-steps 0 2>/dev/null | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print(round(d['ms_per_step'],3), d.get('rounds_rank0'), round(d['node_visits_per_s']/1e6,1))" >> $out
done
timeout 2400 python bench.py --gpus 1 --steps 20 --warmup 5 > gpurun_out/dc_bench_full.jsonl 2> gpurun_out/dc_bench_full.err
