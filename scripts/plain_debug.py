"""PLAIN variant debugging: tiny, random tiny, small; parity vs the oracle."""
import sys, time
import numpy as np
sys.path.insert(0, "."); sys.path.insert(0, "tests/golden")
import torch
import oracle
import paper_conf_ipps_yuwobby20_b200 as gd
from programs import tiny
from synth import random_tiny
from synth import generator as G
which = sys.argv[1] if len(sys.argv) > 1 else "tiny"
gs = {"tiny": lambda: [tiny()[0]], "rand": lambda: [random_tiny(s) for s in range(11000, 11010)],
      "small": lambda: [G.preset("small")]}[which]()
for g in gs:
    app = gd.load(g, plain=True)
    t = time.time()
    st = app.build(variant="plain")
    print(which, g.n_nodes, "plain build ms", st["build_ns"] / 1e6, "rounds", st["rounds"], "visits", st["node_visits"], flush=True)
    per, dig = app.node_digests()
    r = oracle.build_idfg(g)
    print(" digest ok" if dig == r.app_digest else " DIGEST MISMATCH", flush=True)
    ptr, pairs = app.read_all_facts(0)
    print(" facts ok" if np.array_equal(ptr, r.ptr) and np.array_equal(pairs, r.pairs) else " FACTS MISMATCH", flush=True)
    app.free()
