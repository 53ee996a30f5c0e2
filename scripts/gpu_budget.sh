#!/bin/bash
# Narrow batch size sweep (bench.py --node-budget) at HEAD: corpus1000 device step.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/bud_build.log 2>&1
out=gpurun_out/budget.log
: > $out.${TAG:-a}
for b in ${BUDGETS:-16000000 24000000 32000000 16000000 24000000 32000000}; do
  echo "== node_budget $b" >> $out.${TAG:-a}
  timeout 900 python bench.py --steps 3 --warmup 2 --no-cpu-baseline --e2e-steps 1 --no-per-config --node-budget $b 2>/dev/null | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print(round(d['ms_per_step'],1), d['e2e']['value'], d['batch_ms_rank0']['n'], d['parity']['mismatches'][:3])" >> $out.${TAG:-a}
done
