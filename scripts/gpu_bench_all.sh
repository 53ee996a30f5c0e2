# all bench lines for the round's profiles/: corpus (default), median, small, worst, reference arm,
# plus launch list + ncu --set full of k_fixpoint on the default workload.  Usage: gpu_bench_all.sh TAG
TAG=$1
python -c "import __graft_entry__ as g; g.build()" || exit 1
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > gpurun_out/smi_${TAG}.txt
timeout 900 python bench.py 2>&1 | tail -1 > gpurun_out/bench_${TAG}_corpus.json
timeout 600 python bench.py --workload median 2>&1 | tail -1 > gpurun_out/bench_${TAG}_median.json
timeout 600 python bench.py --workload small 2>&1 | tail -1 > gpurun_out/bench_${TAG}_small.json
timeout 900 python bench.py --workload worst --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 2 2>&1 | tail -1 > gpurun_out/bench_${TAG}_worst.json
timeout 600 python bench.py --impl reference --steps 5 --warmup 1 2>&1 | tail -1 > gpurun_out/bench_${TAG}_reference.json
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_${TAG}.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline --e2e-steps 0 > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_fixpoint -c 1 -o gpurun_out/prof_${TAG} python bench.py --steps 1 --warmup 0 --no-cpu-baseline --e2e-steps 0 > gpurun_out/ncu_${TAG}.log 2>&1
ls -la gpurun_out | grep $TAG
