#!/bin/bash
# A/B: dynamic hand-out in narrow rounds with G items per claim (GD_DYN_NARROW=1, GD_DYN_GRAIN=G)
# vs warp-strided narrow items (GD_DYN_NARROW=0).
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
out=gpurun_out/ab_grain.log
: > $out
for v in "1 8" "1 32" "0 8" "1 8" "1 32" "0 8"; do
  set -- $v
  GDROID_NVCC_FLAGS="-DGD_DYN_NARROW=$1 -DGD_DYN_GRAIN=$2" python -c "import __graft_entry__ as g; g.build()" >> gpurun_out/ab_build.log 2>&1
  for w in small median; do
    echo "== NARROW=$1 GRAIN=$2 $w" >> $out
    timeout 600 python bench.py --workload $w --steps 10 --warmup 3 --no-cpu-baseline --e2e-steps 0 2>/dev/null | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print(round(d['ms_per_step'],3), d.get('rounds_rank0'), round(d['node_visits_per_s']/1e6,1))" >> $out
  done
  echo "== NARROW=$1 GRAIN=$2 corpus1000" >> $out
  timeout 900 python bench.py --steps 3 --warmup 2 --no-cpu-baseline --e2e-steps 0 --no-per-config 2>/dev/null | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print(round(d['ms_per_step'],1), d['batch_ms_rank0'], d['parity']['mismatches'][:3])" >> $out
done
GDROID_NVCC_FLAGS="" python -c "import __graft_entry__ as g; g.build()" >> gpurun_out/ab_build.log 2>&1
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/ab_grain_gpu_tests.log 2>&1
