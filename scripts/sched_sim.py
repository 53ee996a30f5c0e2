"""Scheduling-policy experiment (not a test, not the product): BSP rounds and node visits of
the oracle's round-synchronous variant under a policy (oracle_bsp_rounds_policy).  The fixed
point is policy-independent; only rounds and visits change.
usage: python scripts/sched_sim.py median 0 1 2 3:16 3:64 ..."""
import ctypes as C
import os
import sys
import time

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import oracle  # noqa: E402
from oracle import _desc, _ptr, lib  # noqa: E402
from synth.generator import corpus_app, preset  # noqa: E402


def run(g, policy):
    L = lib()
    d, keep = _desc(g)
    seq = np.zeros(1 << 16, dtype=np.uint32)
    lens = np.zeros(1 << 16, dtype=np.uint32)
    v = C.c_uint64(0)
    L.oracle_bsp_rounds_policy.restype = C.c_int64
    nr = L.oracle_bsp_rounds_policy(C.byref(d), policy, _ptr(seq), len(seq), _ptr(lens), len(lens), C.byref(v))
    return nr, v.value, int(seq[:nr].sum()) if (policy & 0xff) in (2, 5) else nr


if __name__ == "__main__":
    w = sys.argv[1]
    g = corpus_app(int(w[6:])) if w.startswith("corpus") else preset(w)
    r = oracle.build_idfg(g, order=3)
    print(f"{w}: nodes {g.n_nodes}  priority-order visits {r.visits / g.n_nodes:.2f}/node")
    for p in sys.argv[2:]:
        pol, _, win = p.partition(":")
        code = int(pol) | (int(win or 0) << 8)
        t = time.time()
        nr, v, cp = run(g, code)
        print(f"policy {p:>8}: rounds {nr:6d}  visits {v / g.n_nodes:6.2f}/node  critical path {cp:6d} items  ({time.time() - t:.1f}s)")
