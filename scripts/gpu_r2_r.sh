python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -1
timeout 900 python -m pytest tests/test_gpu_corpus.py tests/test_gpu_parity.py tests/test_gpu_ooc.py -x -q 2>&1 | tail -1
timeout 900 python scripts/readback_bench.py
timeout 900 python scripts/e2e_diag.py 200
timeout 900 python bench.py --n-apps 200 --steps 1 --warmup 1 --no-per-config --no-cpu-baseline --e2e-steps 1 --e2e-reserve-sms 0 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('reserve 0 corpus200 device', round(d['ms_per_step'],1), 'e2e', round(d['e2e']['ms_per_step'],1))"
timeout 900 python bench.py --n-apps 200 --steps 1 --warmup 1 --no-per-config --no-cpu-baseline --e2e-steps 1 --e2e-reserve-sms 8 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('reserve 8 corpus200 device', round(d['ms_per_step'],1), 'e2e', round(d['e2e']['ms_per_step'],1))"
