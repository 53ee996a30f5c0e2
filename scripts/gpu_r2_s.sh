python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -1
timeout 900 python -m pytest tests/test_gpu_corpus.py -x -q 2>&1 | tail -3
for R in 4 0 8; do
timeout 900 python bench.py --n-apps 200 --steps 1 --warmup 1 --no-per-config --no-cpu-baseline --e2e-steps 2 --e2e-reserve-sms $R 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('reserve $R corpus200 device', round(d['ms_per_step'],1), 'e2e', round(d['e2e']['ms_per_step'],1), round(d['e2e']['d2h_bytes_per_step']/1e9,1))"
done
