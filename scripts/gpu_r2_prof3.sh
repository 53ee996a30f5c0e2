python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:k_fixpoint -c 1 -o gpurun_out/r2_worst_final python bench.py --workload worst --steps 1 --warmup 0 --no-cpu-baseline --e2e-steps 0 --no-per-config > gpurun_out/ncu_r2_worst_final.log 2>&1
tail -1 gpurun_out/ncu_r2_worst_final.log
