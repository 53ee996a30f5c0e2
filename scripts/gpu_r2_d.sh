# CELL variant parity, corpus1000 DRAM bytes of every k_fixpoint launch (ncu, 3 metrics), launch list, ablation
python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -1
timeout 1200 python -m pytest tests/test_gpu_parity.py -x -q -k "cell" 2>&1 | tail -3
timeout 600 python -m pytest tests/test_gpu_fullsize.py -x -q -k "cell" 2>&1 | tail -3
timeout 1800 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r02_corpus1000_launches.csv python bench.py --steps 1 --warmup 0 --no-cpu-baseline --e2e-steps 0 --no-per-config > gpurun_out/r02_ncu_corpus1000.log 2>&1; echo "ncu rc=$?"
tail -c 600 gpurun_out/r02_ncu_corpus1000.log
timeout 1800 python scripts/ablation.py --apps 24 --reps 3 --out gpurun_out/r02_ablation.json 2>&1 | tail -14
