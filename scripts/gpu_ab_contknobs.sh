#!/bin/bash
# Sweep of the continuation knobs at the final kernel: depth (GD_CONT_DEPTH) and the light-round
# threshold (GD_CONT_LOAD: continuation while items < GD_CONT_LOAD/4 x warps).
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
out=gpurun_out/ab_contknobs.log
: > $out
for v in "8 4" "12 4" "8 8" "4 4" "8 4" "12 4" "8 8" "4 4"; do
  set -- $v
  GDROID_NVCC_FLAGS="-DGD_CONT_DEPTH=$1 -DGD_CONT_LOAD=$2" python -c "import __graft_entry__ as g; g.build()" >> gpurun_out/ab_build.log 2>&1
  for w in small median; do
    echo "== DEPTH=$1 LOAD=$2 $w" >> $out
    timeout 600 python bench.py --workload $w --steps 10 --warmup 3 --no-cpu-baseline --e2e-steps 0 2>/dev/null | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print(round(d['ms_per_step'],3), d.get('rounds_rank0'), round(d['node_visits_per_s']/1e6,1))" >> $out
  done
  echo "== DEPTH=$1 LOAD=$2 corpus1000" >> $out
  timeout 900 python bench.py --steps 3 --warmup 2 --no-cpu-baseline --e2e-steps 0 --no-per-config 2>/dev/null | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print(round(d['ms_per_step'],1), d['batch_ms_rank0']['wide'], d['parity']['mismatches'][:3])" >> $out
done
GDROID_NVCC_FLAGS="" python -c "import __graft_entry__ as g; g.build()" >> gpurun_out/ab_build.log 2>&1
