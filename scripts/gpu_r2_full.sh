# round 2: the metric's full workload (corpus1000 on 1 GPU, default bench), out-of-core worst, sanitizers
python -c "import __graft_entry__ as g; g.build()" || exit 1
nvidia-smi --query-gpu=memory.used,memory.total --format=csv
timeout 1800 python bench.py --steps 3 --warmup 2 > gpurun_out/r02_bench_full.jsonl 2> gpurun_out/r02_bench_full.err; echo "bench rc=$?"
tail -c 3000 gpurun_out/r02_bench_full.err
timeout 1200 python scripts/ooc_bench.py worst 4 > gpurun_out/r02_ooc_worst.json 2> gpurun_out/r02_ooc_worst.err; echo "ooc rc=$?"; cat gpurun_out/r02_ooc_worst.json; tail -5 gpurun_out/r02_ooc_worst.err
bash scripts/gpu_r2_sanitize.sh
