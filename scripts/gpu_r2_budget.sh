# batch-size sweep of the corpus path (narrow node budget, wide apps per batch)
python -c "import __graft_entry__ as g; g.build()" || exit 1
for B in 2000000 4000000 8000000 16000000; do
  timeout 900 python bench.py --n-apps 200 --steps 2 --warmup 1 --no-per-config --no-cpu-baseline --e2e-steps 0 --node-budget $B 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('budget $B', round(d['ms_per_step'],1), d['batch_ms_rank0'], d['parity'])"
done
timeout 900 python bench.py --n-apps 200 --steps 2 --warmup 1 --no-per-config --no-cpu-baseline --e2e-steps 0 --wide-per-batch 2 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('wide2', round(d['ms_per_step'],1), d['batch_ms_rank0'])"
