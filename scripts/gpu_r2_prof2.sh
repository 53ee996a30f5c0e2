# ncu --set full of one heavy narrow k_fixpoint launch (4-CTA/SM instantiation) on a 16M-node corpus batch
python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 1500 ncu --set full --clock-control none --import-source on --kernel-name-base mangled -k regex:ILb0ELb0ELi1ELi4 -c 1 -o gpurun_out/r2_narrow_heavy python bench.py --n-apps 40 --steps 1 --warmup 0 --no-cpu-baseline --e2e-steps 0 --no-per-config > gpurun_out/ncu_r2_narrow.log 2>&1
tail -2 gpurun_out/ncu_r2_narrow.log
ls -la gpurun_out/r2_narrow_heavy.ncu-rep
