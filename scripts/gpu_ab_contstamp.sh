#!/bin/bash
# A/B of the light-round continuation hops: GD_CONT_STAMP (one atomicMax claims the continuation;
# 0 = the round-2 stamp load + atomicExch on cont[] + atomicMax) and GD_CONT_PF (prefetch the
# inline successors' records into L1 when continuation is possible).
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
out=gpurun_out/ab_contstamp.log
: > $out
for v in "1 1" "0 0" "1 0" "1 1" "0 0"; do
  set -- $v
  GDROID_NVCC_FLAGS="-DGD_CONT_STAMP=$1 -DGD_CONT_PF=$2" python -c "import __graft_entry__ as g; g.build()" >> gpurun_out/ab_build.log 2>&1
  for w in small median worst; do
    echo "== STAMP=$1 PF=$2 $w" >> $out
    timeout 600 python bench.py --workload $w --steps 10 --warmup 3 --no-cpu-baseline --e2e-steps 0 2>/dev/null | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print(round(d['ms_per_step'],3), d.get('rounds_rank0'), round(d['node_visits_per_s']/1e6,1))" >> $out
  done
  echo "== STAMP=$1 PF=$2 corpus1000" >> $out
  timeout 900 python bench.py --steps 3 --warmup 2 --no-cpu-baseline --e2e-steps 0 --no-per-config 2>/dev/null | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print(round(d['ms_per_step'],1), d.get('rounds_rank0'), round(d['node_visits_per_s']/1e6,1), d['parity']['mismatches'][:3])" >> $out
done
GDROID_NVCC_FLAGS="" python -c "import __graft_entry__ as g; g.build()" >> gpurun_out/ab_build.log 2>&1
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/ab_gpu_tests.log 2>&1
