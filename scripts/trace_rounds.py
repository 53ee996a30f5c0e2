#!/usr/bin/env python3
"""Per-round timing of one build (diagnostics): round duration vs items, barrier floor."""
import sys
import numpy as np
import torch
sys.path.insert(0, ".")
import paper_conf_ipps_yuwobby20_b200 as gd
from synth import generator as G

wl = sys.argv[1] if len(sys.argv) > 1 else "median"
blocks = int(sys.argv[2]) if len(sys.argv) > 2 else 0
if wl == "chain":   # a long NOP chain: one item per round -> barrier + one-item latency
    from synth import IcfgBuilder
    b = IcfgBuilder(n_fields=1); d = b.add_module(); m = b.add_method(d, 0, 2)
    nodes = [b.nop(m) for _ in range(4000)]
    b.chain(b.entry(m), *nodes, b.exit(m)); b.add_entry(m); gs = [b.build()]
elif wl == "corpus27":
    gs = [G.corpus_app(27)]
elif wl == "corpus8":
    gs = [G.corpus_app(i) for i in range(8)]
else:
    gs = [G.preset(wl)]
app = gd.load(gs, stream=torch.cuda.current_stream().cuda_stream)
app.set_trace(1 << 16)
for _ in range(3):
    st = app.build(blocks=blocks)
tr = app.read_trace()
ph = app.phases().astype(float)
if ph[4] > 0:
    tot = ph[:4].sum()
    print(f"phases (GD_PHASES): items {ph[4]:.0f}  setup {ph[0]/tot:.1%}  edges {ph[1]/tot:.1%}  push {ph[2]/tot:.1%}  "
          f"round-end {ph[3]/tot:.1%};  cycles/item setup {ph[0]/ph[4]:.0f} edges {ph[1]/ph[4]:.0f} push {ph[2]/ph[4]:.0f}")
dt = np.diff(tr[:, 0].astype(np.int64)) / 1e3   # us per round
items = tr[:-1, 1]
print(f"{wl}: rounds {len(dt)} fixpoint {st['fixpoint_ns']/1e6:.3f} ms, mean round {dt.mean():.2f} us, "
      f"queued items {int(items.sum())} node visits {st['node_visits']}")
for lo, hi in [(0, 1), (1, 32), (32, 256), (256, 1024), (1024, 4096), (4096, 16384), (16384, 1 << 30)]:
    m = (items > lo) & (items <= hi) if lo else (items <= hi)
    if m.any():
        print(f"  items in ({lo},{hi}]: rounds {m.sum():5d}  mean {dt[m].mean():8.2f} us  p90 {np.percentile(dt[m], 90):8.2f}  "
              f"share {dt[m].sum() / dt.sum():.2%}  us/item {dt[m].sum() / items[m].sum():.3f}")
