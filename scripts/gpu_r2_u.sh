python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_ooc.py tests/test_gpu_corpus.py -x -q 2>&1 | tail -1
timeout 900 python -m pytest tests/test_gpu_fullsize.py -x -q -k "worst or cell or corpus_wide" 2>&1 | tail -1
timeout 900 python bench.py --n-apps 200 --steps 2 --warmup 1 --no-per-config --no-cpu-baseline --e2e-steps 0 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('corpus200', round(d['ms_per_step'],1), 'fix', round(d['fixpoint_ms_per_step_rank0'],1), 'wide', round(d['batch_ms_rank0']['wide'],1), d['parity'])"
timeout 600 python bench.py --workload worst --steps 3 --warmup 1 --no-cpu-baseline --e2e-steps 0 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('worst', round(d['ms_per_step'],2), 'fix', round(d['fixpoint_ms_per_step_rank0'],2))"
