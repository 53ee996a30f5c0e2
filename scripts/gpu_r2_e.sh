# SBDA parity + timings; PRE/PRE2 A/B on corpus200 with 16M-node batches
python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -1
timeout 1200 python -m pytest tests/test_gpu_parity.py -x -q -k "sbda" 2>&1 | tail -3
timeout 900 python -m pytest tests/test_gpu_fullsize.py -x -q -k "sbda" 2>&1 | tail -3
python - <<'PY'
import json, statistics, paper_conf_ipps_yuwobby20_b200 as gd
from synth import generator as G
for name in ("small", "median", "worst"):
    g = G.preset(name); a = gd.load(g)
    for v in ("default", "sbda"):
        a.build(variant=v, byte_model=False)
        st = [a.build(variant=v, byte_model=False) for _ in range(3)]
        print(name, v, "ms", round(statistics.median(s["build_ns"] for s in st) / 1e6, 3), "rounds", st[-1]["rounds"], "visits", st[-1]["node_visits"])
    a.free()
PY
for F in "" "-DGD_PRE2=0" "-DGD_PRE=0"; do
  GDROID_NVCC_FLAGS="$F" python -c "import __graft_entry__ as g; g.build()" || exit 1
  timeout 900 python bench.py --n-apps 200 --steps 2 --warmup 1 --no-per-config --no-cpu-baseline --e2e-steps 0 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('flags [$F]', round(d['ms_per_step'],1), d['batch_ms_rank0']['wide'], d['parity']['mismatches'])"
done
python -c "import __graft_entry__ as g; g.build()"
