# ncu --set full of k_fixpoint (Δ wide path on worst; narrow corpus8) + source pages
python -c "import __graft_entry__ as g; g.build()" || exit 1
for W in worst corpus8; do
  timeout 1200 ncu --set full --clock-control none --import-source on -k regex:k_fixpoint -c 1 -o gpurun_out/r2_$W python bench.py --workload $W --steps 1 --warmup 0 --no-cpu-baseline --e2e-steps 0 --no-per-config > gpurun_out/ncu_r2_$W.log 2>&1
  tail -1 gpurun_out/ncu_r2_$W.log
  ncu -i gpurun_out/r2_$W.ncu-rep --page source --csv --print-source sass > gpurun_out/r2_${W}_src.csv 2>/dev/null
  ncu -i gpurun_out/r2_$W.ncu-rep --page raw --csv > gpurun_out/r2_${W}_raw.csv 2>/dev/null
done
ls -la gpurun_out
