#!/usr/bin/env python3
"""Write tests/golden/oracle_digests.json: oracle results (ONLY oracle/ computes them) for the
generated configs at full size, used by the GPU parity tests at BASELINE.json's sizes.

Per config: generator version + preset, node/edge counts, the app digest, an
order-sensitive hash of the per-node digest array, oracle visits/seconds, and the full pair
lists of 24 sampled nodes (seeded choice, biased to non-empty sets).
"""
import json
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import oracle  # noqa: E402
from synth import generator as G  # noqa: E402

OUT = os.path.join(ROOT, "tests", "golden", "oracle_digests.json")
M = (1 << 64) - 1


def mix64(z):
    z &= M
    z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & M
    z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & M
    return z ^ (z >> 31)


def node_hash(per_node):
    h = 0
    for i, d in enumerate(per_node.tolist()):
        h = (h + mix64((i * 0x9E3779B97F4A7C15) ^ d)) & M
    return h


def entry(name, g):
    t = time.time()
    r = oracle.build_idfg(g)
    rng = np.random.default_rng(12345)
    sizes = np.diff(r.ptr.astype(np.int64))
    nonempty = np.nonzero(sizes)[0]
    pick = sorted(set(rng.choice(nonempty, size=min(20, len(nonempty)), replace=False).tolist())
                  | set(rng.choice(g.n_nodes, size=4, replace=False).tolist()))
    return {"name": name, "gen_version": G.GEN_VERSION, "n_nodes": g.n_nodes, "n_edges": g.n_edges,
            "app_digest": str(r.app_digest), "node_digest_hash": str(node_hash(r.node_digest)),
            "visits": r.visits, "oracle_s": r.seconds, "wall_s": time.time() - t,
            "samples": {str(n): [str(int(p)) for p in r.facts(n)] for n in pick}}


def main():
    which = sys.argv[1:] or ["small", "median", "corpus16", "worst"]
    data = json.load(open(OUT)) if os.path.exists(OUT) else {}
    for w in which:
        if w == "corpus16":
            for i in range(16):
                key = f"corpus{i}"
                data[key] = entry(key, G.corpus_app(i))
                print(key, data[key]["n_nodes"], data[key]["oracle_s"], flush=True)
        else:
            data[w] = entry(w, G.preset(w))
            print(w, data[w]["n_nodes"], data[w]["oracle_s"], flush=True)
        json.dump(data, open(OUT, "w"), indent=0)


if __name__ == "__main__":
    main()
