python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "hybrid or heavy_round" 2>&1 | grep -E "Error|error|assert|Exception|passed|failed" | head -20
timeout 900 python -m pytest tests/test_gpu_fullsize.py -x -q -k "median or corpus_digest_sample" 2>&1 | tail -1
for F in "" "-DGD_PAIR=0"; do
  GDROID_NVCC_FLAGS="$F" python -c "import __graft_entry__ as g; g.build()" || exit 1
  timeout 900 python bench.py --n-apps 200 --steps 2 --warmup 1 --no-per-config --no-cpu-baseline --e2e-steps 0 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('[$F] corpus200', round(d['ms_per_step'],1), 'wide', round(d['batch_ms_rank0']['wide'],1), d['parity']['mismatches'])"
  timeout 600 python bench.py --workload median --steps 5 --warmup 2 --no-cpu-baseline --e2e-steps 0 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('[$F] median', round(d['ms_per_step'],3), d['rounds_rank0'])"
done
python -c "import __graft_entry__ as g; g.build()"
