# per-round traces for kernel variants: bash scripts/gpu_trace2.sh "<flags>" ...
for v in "$@"; do
  GDROID_NVCC_FLAGS="$v" python -c "import paper_conf_ipps_yuwobby20_b200._build as b; b.build()" || exit 1
  for w in chain median corpus8 worst; do echo "== [$v]"; timeout 300 python scripts/trace_rounds.py $w 2>&1 | tail -9; done
done
