# 3-CTA/SM instantiation with continuation for every narrow batch (never the 4-CTA one), continuation in light / all rounds
for F in "-DGD_HIOCC_NODES=4000000000u" "-DGD_HIOCC_NODES=4000000000u -DGD_CONT_LOAD=100000000"; do
  GDROID_NVCC_FLAGS="$F" python -c "import __graft_entry__ as g; g.build()" || exit 1
  timeout 900 python bench.py --n-apps 200 --steps 2 --warmup 1 --no-per-config --no-cpu-baseline --e2e-steps 0 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('[$F] corpus200', round(d['ms_per_step'],1), 'wide', round(d['batch_ms_rank0']['wide'],1), 'visits/s', round(d['node_visits_per_s']/1e6), 'visits', round(d['node_visits_per_s']*d['ms_per_step']/1e9,1), 'M', d['parity']['mismatches'])"
  timeout 600 python bench.py --workload median --steps 5 --warmup 2 --no-cpu-baseline --e2e-steps 0 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('[$F] median', round(d['ms_per_step'],3), d['rounds_rank0'])"
done
python -c "import __graft_entry__ as g; g.build()"
