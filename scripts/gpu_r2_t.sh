# A/B: wide instantiation at 4 CTAs/SM; hybrid heavy-round threshold at 16M-node batches
for F in "" "-DGD_MINB_WIDE=4" "-DGD_HYB_HI=8" "-DGD_HYB_HI=32"; do
  GDROID_NVCC_FLAGS="$F" python -c "import __graft_entry__ as g; g.build()" || exit 1
  timeout 600 python bench.py --workload worst --steps 3 --warmup 1 --no-cpu-baseline --e2e-steps 0 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('[$F] worst', round(d['ms_per_step'],2), d['rounds_rank0'])"
  timeout 900 python bench.py --n-apps 200 --steps 2 --warmup 1 --no-per-config --no-cpu-baseline --e2e-steps 0 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('[$F] corpus200', round(d['ms_per_step'],1), 'wide', round(d['batch_ms_rank0']['wide'],1), d['parity']['mismatches'])"
done
python -c "import __graft_entry__ as g; g.build()"
