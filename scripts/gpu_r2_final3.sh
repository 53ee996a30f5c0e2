#!/bin/bash
# Round-2 closing measurements at HEAD (session 3, final): smoke, GPU suite, default bench + reference
# arm, ncu launch list / DRAM traffic of one corpus1000 step, ncu --set full of one heavy narrow
# launch, device-layout load timing.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/f3_smoke.log 2>&1; tail -1 gpurun_out/f3_smoke.log
( time timeout 3000 python -m pytest tests -m gpu -q ) > gpurun_out/f3_gpu_tests.log 2>&1; tail -4 gpurun_out/f3_gpu_tests.log
timeout 2400 python bench.py --steps 5 --warmup 3 > gpurun_out/f3_bench.jsonl 2> gpurun_out/f3_bench.err; echo "bench rc=$?"
timeout 1200 python bench.py --impl reference --steps 5 --warmup 1 >> gpurun_out/f3_bench.jsonl 2>> gpurun_out/f3_bench.err; echo "ref rc=$?"
GDROID_TIMING=1 timeout 600 python scripts/load_timing.py 60 > gpurun_out/f3_load_dev.log 2>&1
timeout 2400 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/f3_corpus1000_launches.csv python bench.py --steps 1 --warmup 0 --no-cpu-baseline --e2e-steps 0 --no-per-config > /dev/null 2>&1; echo "ncu rc=$?"
BUILDS=1 timeout 1500 ncu --set full --clock-control none --import-source on --kernel-name-base demangled \
  -k "regex:k_fixpoint.*\(int\)4>" -c 1 -o gpurun_out/f3_heavy python scripts/heavy_batch.py > gpurun_out/f3_ncu_heavy.log 2>&1; echo "ncu heavy rc=$?"
ncu -i gpurun_out/f3_heavy.ncu-rep --page raw --csv > gpurun_out/f3_heavy_raw.csv 2>/dev/null
rm -f gpurun_out/f3_heavy.ncu-rep
