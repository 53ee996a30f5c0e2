# build each variant, then bench median/corpus/worst
# usage: bash scripts/gpu_variants.sh "<nvcc flags>|<env assignments>" ...
mkdir -p gpurun_out
for v in "$@"; do
  flags="${v%%|*}"; envs=""; [[ "$v" == *"|"* ]] && envs="${v#*|}"
  GDROID_NVCC_FLAGS="-DGD_AB $flags" python -c "import paper_conf_ipps_yuwobby20_b200._build as b; b.build()" || exit 1
  for w in ${WORKLOADS:-median corpus worst}; do
    echo "== [$flags] [$envs] $w"
    env $envs timeout 600 python bench.py --workload $w --steps 5 --warmup 3 --no-cpu-baseline --e2e-steps 1 2>&1 | tail -1 | \
      python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['ms_per_step'], d['rounds_per_step'], round(d['node_visits_per_s']*d['ms_per_step']/1e3), d['config']['nodes_per_rank'])"
  done
done
