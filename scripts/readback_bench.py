#!/usr/bin/env python3
"""Raw speed of gdroid_read_batch_facts on one built 16M-node corpus batch (no concurrent build):
popc + D2H counts + prefix + H2D ptr + expand + D2H pairs into pinned buffers."""
import os, sys, time
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch
import paper_conf_ipps_yuwobby20_b200 as gd
from paper_conf_ipps_yuwobby20_b200 import corpus
from synth import generator as G
n = 60
sizes = G.corpus_sizes(n)
wide = [G.corpus_config(i).q_cap > 64 for i in range(n)]
plan = corpus.plan_corpus(sizes, wide, 1, node_budget=16_000_000)
b = [x for x in plan.batches[0] if not wide[x[0]]][0]
apps = corpus.make_apps(b, G.corpus_app, threads=16)
h = gd.load([apps[i] for i in b])
h.build()
bufs = corpus.ReadbackBuffers()
h.read_batch_facts(bufs.ptr, bufs.pairs)
for rep in range(3):
    torch.cuda.synchronize(); t = time.perf_counter()
    ptr, pairs = h.read_batch_facts(bufs.ptr, bufs.pairs)
    dt = time.perf_counter() - t
    print(f"batch {len(b)} apps {sum(h.n_nodes)} nodes: {pairs.nbytes/1e9:.2f} GB pairs in {dt*1e3:.1f} ms = {pairs.nbytes/dt/1e9:.1f} GB/s")
