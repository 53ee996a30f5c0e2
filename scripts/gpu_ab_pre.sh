#!/bin/bash
# A/B: IN(dst) pre-reads of inline items with 3 words per lane (GD_PRE / GD_PRE2), and the e2e
# timeline with fact vs digest readback (what slows builds inside the pipeline).
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
out=gpurun_out/ab_pre.log
: > $out
for v in "1 1" "1 0" "0 0" "1 1" "1 0" "0 0"; do
  set -- $v
  GDROID_NVCC_FLAGS="-DGD_PRE=$1 -DGD_PRE2=$2" python -c "import __graft_entry__ as g; g.build()" >> gpurun_out/ab_build.log 2>&1
  for w in small median; do
    echo "== PRE=$1 PRE2=$2 $w" >> $out
    timeout 600 python bench.py --workload $w --steps 10 --warmup 3 --no-cpu-baseline --e2e-steps 0 2>/dev/null | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print(round(d['ms_per_step'],3), d.get('rounds_rank0'), round(d['node_visits_per_s']/1e6,1))" >> $out
  done
  echo "== PRE=$1 PRE2=$2 corpus1000" >> $out
  timeout 900 python bench.py --steps 3 --warmup 2 --no-cpu-baseline --e2e-steps 0 --no-per-config 2>/dev/null | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print(round(d['ms_per_step'],1), d['batch_ms_rank0'], d['parity']['mismatches'][:3])" >> $out
done
GDROID_NVCC_FLAGS="" python -c "import __graft_entry__ as g; g.build()" >> gpurun_out/ab_build.log 2>&1
timeout 1200 python scripts/e2e_timeline.py 1000 facts > gpurun_out/tl_facts.jsonl 2> gpurun_out/tl_facts.err
timeout 1200 python scripts/e2e_timeline.py 1000 digests > gpurun_out/tl_digests.jsonl 2> gpurun_out/tl_digests.err
