python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
python - <<'PY'
import statistics, paper_conf_ipps_yuwobby20_b200 as gd
from synth import generator as G
for name in ("small", "median"):
    g = G.preset(name); a = gd.load(g)
    for blocks in (0, 74, 148, 296):
        a.build(blocks=blocks, byte_model=False)
        st = [a.build(blocks=blocks, byte_model=False) for _ in range(5)]
        print(name, "blocks", blocks or "max", "ms", round(statistics.median(s["build_ns"] for s in st) / 1e6, 3), "rounds", st[-1]["rounds"])
    a.free()
PY
