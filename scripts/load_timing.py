#!/usr/bin/env python3
"""Host-side load phases of gdroid_load_batch (GDROID_TIMING=1 prints them to stderr).
usage: load_timing.py N            corpus apps 0..N-1 in one batch
       load_timing.py app:I        corpus app I alone (per-phase breakdown)"""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ipps_yuwobby20_b200 as gd
from synth import generator as G
arg = sys.argv[1] if len(sys.argv) > 1 else "8"
ids = [int(arg[4:])] if arg.startswith("app:") else list(range(int(arg)))
gs = [G.corpus_app(i) for i in ids]
print(f"apps {ids}: {sum(g.n_nodes for g in gs)} nodes", file=sys.stderr)
for it in range(4):
    t = time.perf_counter()
    a = gd.load(gs, stream=torch.cuda.current_stream().cuda_stream)
    t1 = time.perf_counter()
    a.free()
    torch.cuda.synchronize()
    print(f"--- iteration {it}: load {1e3 * (t1 - t):.1f} ms, free {1e3 * (time.perf_counter() - t1):.1f} ms", file=sys.stderr, flush=True)
