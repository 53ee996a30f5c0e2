#!/usr/bin/env python3
"""Timeline of the end-to-end corpus pipeline (corpus.run_pipelined): per batch, when its load
started / returned (loader thread), when its build was enqueued and its sync returned, and when
its fact readback was enqueued / completed (wraps the binding calls from outside)."""
import os, sys, time, json
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch
import paper_conf_ipps_yuwobby20_b200 as gd
from paper_conf_ipps_yuwobby20_b200 import corpus, _binding
from synth import generator as G

n = int(sys.argv[1]) if len(sys.argv) > 1 else 1000
readback = sys.argv[2] if len(sys.argv) > 2 else "facts"
sizes = G.corpus_sizes(n)
wide = [G.corpus_config(i).q_cap > 64 for i in range(n)]
plan = corpus.plan_corpus(sizes, wide, 1, node_budget=16_000_000)
apps = corpus.make_apps(plan.shards[0], G.corpus_app, threads=16)
EV = []
T0 = [0.0]
def now(): return round((time.perf_counter() - T0[0]) * 1e3, 2)
orig = {k: getattr(_binding.App, k) for k in ("build", "sync", "read_batch_facts_async", "stream_sync", "free")}
orig_load = _binding.load
def w_load(*a, **k):
    t = now(); r = orig_load(*a, **k); EV.append(("load", id(r), t, now(), sum(x.n_nodes for x in a[0]))); return r
def wrap(name):
    f = orig[name]
    def g(self, *a, **k):
        t = now(); r = f(self, *a, **k); EV.append((name, id(self), t, now(), 0)); return r
    return g
_binding.load = w_load
for k in orig: setattr(_binding.App, k, wrap(k))
bufs = corpus.ReadbackBuffers()
corpus.run_pipelined(plan.batches[0], lambda i: apps[i], bufs=bufs, readback=readback)   # warm-up (sizes buffers)
EV.clear()
torch.cuda.synchronize()
T0[0] = time.perf_counter()
res = corpus.run_pipelined(plan.batches[0], lambda i: apps[i], bufs=bufs, readback=readback)
wall = now()
build_dev_ms = sum(r.stats["build_ns"] for r in res) / 1e6
ids = {}
rows = []
for ev in EV:
    b = ids.setdefault(ev[1], len(ids))
    rows.append({"batch": b, "ev": ev[0], "t0": ev[2], "t1": ev[3], "nodes": ev[4]})
tot = {}
for r in rows:
    tot[r["ev"]] = round(tot.get(r["ev"], 0) + r["t1"] - r["t0"], 1)
print(json.dumps({"wall_ms": wall, "readback": readback, "batches": len(plan.batches[0]), "sum_ms": tot,
                  "build_device_ms": round(build_dev_ms, 1)}))
for r in rows:
    print(json.dumps(r))
