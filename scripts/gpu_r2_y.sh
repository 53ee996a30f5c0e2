# continuation in the 4-CTA/SM heavy-round build (GD_CD_HI), in light rounds only / in every round
for F in "-DGD_CD_HI=1" "-DGD_CD_HI=1 -DGD_CONT_LOAD=100000000" "-DGD_CD_HI=1 -DGD_CONT_LOAD=32"; do
  GDROID_NVCC_FLAGS="$F" python -c "import __graft_entry__ as g; g.build()" || exit 1
  grep -A2 "k_fixpointILb0ELb0ELi1ELi4" paper_conf_ipps_yuwobby20_b200/ptxas_info.txt | grep spill | head -1
  timeout 900 python bench.py --n-apps 200 --steps 2 --warmup 1 --no-per-config --no-cpu-baseline --e2e-steps 0 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('[$F] corpus200', round(d['ms_per_step'],1), 'wide', round(d['batch_ms_rank0']['wide'],1), 'visits', round(d['node_visits_per_s']*d['ms_per_step']/1e9,1), 'M', d['parity']['mismatches'])"
  timeout 600 python bench.py --workload median --steps 5 --warmup 2 --no-cpu-baseline --e2e-steps 0 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('[$F] median', round(d['ms_per_step'],3), d['rounds_rank0'])"
done
python -c "import __graft_entry__ as g; g.build()"
