#!/usr/bin/env python3
"""Out-of-core sub-graph streaming on a preset: solve with K
sub-graphs (at most two fact stores on the device, dual-buffered imports), time it against the
in-core build, and check the result's app digest (C8, recomputed on the host from the read-back
pairs with the ORIGINAL node ids) against the stored oracle digest.

usage: ooc_bench.py [preset=worst] [K=4]  -> one JSON line
"""
import json
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import paper_conf_ipps_yuwobby20_b200 as gd  # noqa: E402
from paper_conf_ipps_yuwobby20_b200 import ooc  # noqa: E402
from synth import generator as G  # noqa: E402


def mix64(z):
    with np.errstate(over="ignore"):
        z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
        z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
        return z ^ (z >> np.uint64(31))


def app_digest(ptr, pairs, chunk=1 << 26):
    """Σ_n Σ_{p in IN(n)} mix64(mix64(n) ^ p) mod 2^64, chunked."""
    cnt = np.diff(ptr.astype(np.int64))
    node = np.repeat(np.arange(len(cnt), dtype=np.uint64), cnt)
    tot = np.uint64(0)
    with np.errstate(over="ignore"):
        for a in range(0, len(pairs), chunk):
            tot += mix64(mix64(node[a:a + chunk]) ^ pairs[a:a + chunk]).sum(dtype=np.uint64)
    return int(tot)


def main():
    import torch
    name = sys.argv[1] if len(sys.argv) > 1 else "worst"
    K = int(sys.argv[2]) if len(sys.argv) > 2 else 4
    g = G.preset(name)
    ref = json.load(open(os.path.join(ROOT, "tests", "golden", "oracle_digests.json"))).get(name, {})
    # in-core reference time
    app = gd.load(g)
    app.build(byte_model=False)
    st = app.build(byte_model=False)
    incore_ms = st["build_ns"] / 1e6
    incore_bytes = app.fact_bytes
    app.free()
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    o = ooc.OutOfCore(g, K)
    setup_s = time.perf_counter() - t0
    s = o.run()
    ptr, pairs = o.read_all_facts()
    dig = app_digest(ptr, pairs)
    line = {"preset": name, "nodes": g.n_nodes, "parts": K,
            "ooc_s": s.seconds, "setup_s": setup_s, "sweeps": s.sweeps, "solves": s.solves,
            "rounds": s.rounds, "visits": s.visits, "device_build_ms": s.build_ms,
            "h2d_gb": s.h2d_bytes / 1e9, "d2h_gb": s.d2h_bytes / 1e9, "seed_pairs": s.seeds,
            "fact_store_gb_total": sum(h.fact_bytes for h in o.handles) / 1e9,
            "peak_resident_fact_gb": s.peak_resident_fact_bytes / 1e9,
            "incore_fact_store_gb": incore_bytes / 1e9, "incore_build_ms": incore_ms,
            "app_digest": str(dig), "oracle_app_digest": ref.get("app_digest"),
            "parity": "ok" if ref and str(dig) == ref["app_digest"] else "MISMATCH" if ref else "no cache"}
    o.free()
    print(json.dumps(line), flush=True)


if __name__ == "__main__":
    main()
