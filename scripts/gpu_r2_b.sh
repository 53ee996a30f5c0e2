# round 2: Δ wide path — parity (wide pools, presets) + worst/corpus timings
python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -2
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_corpus.py tests/test_gpu_generated.py -x -q 2>&1 | tail -4
timeout 600 python -m pytest tests/test_gpu_fullsize.py -x -q -k "small or median or batches_full or run_shard" 2>&1 | tail -4
timeout 600 python bench.py --workload worst --steps 3 --warmup 1 --no-cpu-baseline --e2e-steps 0 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('worst', d['ms_per_step'], d['rounds_rank0'], d['node_visits_per_s'], d['roofline']['frac'])"
timeout 900 python bench.py --n-apps 100 --steps 2 --warmup 1 --no-per-config --no-cpu-baseline 2>&1 | tail -1
