#!/bin/bash
# Narrow continuation depth sweep (GD_CONT_DEPTH_NARROW) at HEAD.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
out=gpurun_out/ab_depthn.log
: > $out
for v in 2 3 4 2 3 4; do
  GDROID_NVCC_FLAGS="-DGD_CONT_DEPTH_NARROW=$v" python -c "import __graft_entry__ as g; g.build()" >> gpurun_out/ab_build.log 2>&1
  for w in small median; do
    echo "== DEPTH_NARROW=$v $w" >> $out
    timeout 600 python bench.py --workload $w --steps 10 --warmup 3 --no-cpu-baseline --e2e-steps 0 2>/dev/null | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print(round(d['ms_per_step'],3), d.get('rounds_rank0'), round(d['node_visits_per_s']/1e6,1))" >> $out
  done
  echo "== DEPTH_NARROW=$v corpus1000" >> $out
  timeout 900 python bench.py --steps 3 --warmup 2 --no-cpu-baseline --e2e-steps 0 --no-per-config 2>/dev/null | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print(round(d['ms_per_step'],1), d['batch_ms_rank0']['wide'], d['parity']['mismatches'][:3])" >> $out
done
GDROID_NVCC_FLAGS="" python -c "import __graft_entry__ as g; g.build()" >> gpurun_out/ab_build.log 2>&1
