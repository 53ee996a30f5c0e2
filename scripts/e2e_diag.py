#!/usr/bin/env python3
"""Where the end-to-end corpus time goes: loader (host tables + H2D), consumer waits, builds,
fact readback — run_pipelined instrumented from outside (wraps the binding calls)."""
import os, sys, time
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch
import paper_conf_ipps_yuwobby20_b200 as gd
from paper_conf_ipps_yuwobby20_b200 import corpus, _binding
from synth import generator as G

n = int(sys.argv[1]) if len(sys.argv) > 1 else 200
sizes = G.corpus_sizes(n)
wide = [G.corpus_config(i).q_cap > 64 for i in range(n)]
plan = corpus.plan_corpus(sizes, wide, 1, node_budget=16_000_000)
apps = corpus.make_apps(plan.shards[0], G.corpus_app, threads=16)
T = {"load": 0.0, "build_sync": 0.0, "readback": 0.0, "digests": 0.0}
orig_load, orig_sync, orig_rb, orig_dig = _binding.load, _binding.App.sync, _binding.App.read_batch_facts, _binding.App.app_digests
def tl(*a, **k):
    t = time.perf_counter(); r = orig_load(*a, **k); T["load"] += time.perf_counter() - t; return r
def ts(self):
    t = time.perf_counter(); r = orig_sync(self); T["build_sync"] += time.perf_counter() - t; return r
def trb(self, *a, **k):
    t = time.perf_counter(); r = orig_rb(self, *a, **k); T["readback"] += time.perf_counter() - t; return r
def td(self):
    t = time.perf_counter(); r = orig_dig(self); T["digests"] += time.perf_counter() - t; return r
_binding.load = tl; _binding.App.sync = ts; _binding.App.read_batch_facts = trb; _binding.App.app_digests = td
bufs = corpus.ReadbackBuffers()
corpus.run_pipelined(plan.batches[0], lambda i: apps[i], bufs=bufs)
for k in T: T[k] = 0.0
torch.cuda.synchronize()
t0 = time.perf_counter()
out = corpus.run_pipelined(plan.batches[0], lambda i: apps[i], bufs=bufs)
wall = time.perf_counter() - t0
print({"apps": n, "batches": len(plan.batches[0]), "wall_s": round(wall, 3), **{k: round(v, 3) for k, v in T.items()},
       "d2h_gb": round(sum(b.d2h_bytes for b in out) / 1e9, 2), "h2d_gb": round(sum(b.h2d_bytes for b in out) / 1e9, 2)})
