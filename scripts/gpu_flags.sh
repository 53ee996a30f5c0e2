# A/B of compile-time kernel switches on one box: parity tests on the default build, then
# bench ms/step per flag set.  usage: bash scripts/gpu_flags.sh "<flags>" ...   ("" = default)
python -c "import __graft_entry__ as g; g.build()" || exit 1
[ -z "$NOTEST" ] && (timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -3)
for rep in 1 2; do
  for v in "$@"; do
    GDROID_NVCC_FLAGS="-DGD_AB $v" python -c "import paper_conf_ipps_yuwobby20_b200._build as b; b.build()"
    for w in ${WORKLOADS:-small median corpus}; do
      printf "[%s] %s: " "$v" "$w"
      timeout 600 python bench.py --workload $w --steps 5 --warmup 3 --no-cpu-baseline --e2e-steps 0 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['ms_per_step'],3), d['rounds_per_step'], round(d['roofline']['frac'],4))"
    done
  done
done
