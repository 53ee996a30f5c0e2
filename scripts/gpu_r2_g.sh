# round header per CTA: parity + timings; multi-rank bench path on one GPU (gloo); reference arm
python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -1
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_ooc.py -x -q 2>&1 | tail -2
timeout 900 python bench.py --n-apps 200 --steps 2 --warmup 1 --no-per-config --no-cpu-baseline --e2e-steps 0 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('corpus200', round(d['ms_per_step'],1), 'fix', round(d['fixpoint_ms_per_step_rank0'],1), d['parity']['mismatches'])"
timeout 600 python bench.py --workload worst --steps 3 --warmup 1 --no-cpu-baseline --e2e-steps 0 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('worst', round(d['ms_per_step'],2), d['rounds_rank0'])"
timeout 600 python bench.py --workload median --steps 5 --warmup 2 --no-cpu-baseline --e2e-steps 0 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('median', round(d['ms_per_step'],3), d['rounds_rank0'])"
GDROID_BENCH_SHARE_GPU=1 timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --n-apps 60 --steps 2 --warmup 1 --no-per-config --cpu-seconds 3 > gpurun_out/r02_two_rank.log 2>&1; echo "two-rank rc=$?"; tail -c 1500 gpurun_out/r02_two_rank.log
timeout 900 python bench.py --impl reference --steps 3 --warmup 1 2>&1 | tail -1
