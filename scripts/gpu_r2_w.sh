# two-stage prefetch pipeline (GD_PF) A/B
python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -1
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q 2>&1 | tail -1
for F in "" "-DGD_PF=0"; do
  GDROID_NVCC_FLAGS="$F" python -c "import __graft_entry__ as g; g.build()" || exit 1
  for i in 1 2; do
  timeout 900 python bench.py --n-apps 200 --steps 2 --warmup 1 --no-per-config --no-cpu-baseline --e2e-steps 0 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('[$F] corpus200', round(d['ms_per_step'],1), 'fix', round(d['fixpoint_ms_per_step_rank0'],1), 'wide', round(d['batch_ms_rank0']['wide'],1), d['parity']['mismatches'])"
  done
  timeout 600 python bench.py --workload median --steps 5 --warmup 2 --no-cpu-baseline --e2e-steps 0 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('[$F] median', round(d['ms_per_step'],3), d['rounds_rank0'])"
  timeout 600 python bench.py --workload worst --steps 3 --warmup 1 --no-cpu-baseline --e2e-steps 0 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('[$F] worst', round(d['ms_per_step'],2))"
done
python -c "import __graft_entry__ as g; g.build()"
