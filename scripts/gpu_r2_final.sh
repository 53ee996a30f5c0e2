# round-2 closing measurements at HEAD: full GPU suite, default bench, reference arm, ncu traffic of the corpus step
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/r02_final_smoke.log 2>&1; tail -1 gpurun_out/r02_final_smoke.log
( time timeout 3000 python -m pytest tests -m gpu -q ) > gpurun_out/r02_final_gpu_tests.log 2>&1; tail -4 gpurun_out/r02_final_gpu_tests.log
timeout 2400 python bench.py --steps 5 --warmup 3 > gpurun_out/r02_final_bench.jsonl 2> gpurun_out/r02_final_bench.err; echo "bench rc=$?"
timeout 1200 python bench.py --impl reference --steps 5 --warmup 1 >> gpurun_out/r02_final_bench.jsonl 2>> gpurun_out/r02_final_bench.err; echo "ref rc=$?"
timeout 2400 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r02_final_corpus1000_launches.csv python bench.py --steps 1 --warmup 0 --no-cpu-baseline --e2e-steps 0 --no-per-config > /dev/null 2>&1; echo "ncu rc=$?"
