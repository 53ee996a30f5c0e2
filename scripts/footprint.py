#!/usr/bin/env python3
"""Fact-store footprint of the MAT layout variants (Fig. 10
PAPER.md:1237-1253), from the GPU path's own results (not a test, not the product):

  node-major   this repo's store: per node (L_m + n_glob) rows x W words, 32-byte aligned
               (+ row-occupancy words for wide blocks) — the device's fact_bytes
  cell-major   the paper's per-method matrix: |P_m| x |Q_m| cells of an n_m-bit statement mask,
               rounded to 64-bit words per cell
  row-sparse   only non-empty rows: per node a row-pointer word, per stored row a 4-byte row id
               + W words (a hierarchical / sparse-row layout)
  set (tight)  8 bytes per (slot, instance) pair

usage: python scripts/footprint.py [n_apps=8] [--out gpurun_out/footprint.json]
"""
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def layout_sizes(g):
    """(|P_m|, |Q_m|, W_m) per method from the input pools."""
    nf = np.diff(g.type_field_ptr.astype(np.int64))
    heap = np.where(g.inst_type >= 0, nf[np.maximum(g.inst_type, 0)], 0)
    ip = g.module_inst_ptr.astype(np.int64)
    sp = g.module_static_ptr.astype(np.int64)
    D = len(ip) - 1
    q = np.diff(ip)
    glob = np.diff(sp) + np.array([heap[g.module_insts[ip[d]:ip[d + 1]]].sum() for d in range(D)])
    mod = g.method_module.astype(np.int64)
    P = g.method_n_locals.astype(np.int64) + glob[mod]
    Q = q[mod]
    W = np.maximum(1, 2 ** np.ceil(np.log2(np.maximum(1, (Q + 63) // 64)))).astype(np.int64)
    return P, Q, W


def main():
    import torch
    import paper_conf_ipps_yuwobby20_b200 as gd
    from synth import generator as G
    n = int(sys.argv[1]) if len(sys.argv) > 1 and sys.argv[1].isdigit() else 8
    out = sys.argv[sys.argv.index("--out") + 1] if "--out" in sys.argv else None
    sizes = G.corpus_sizes(1000)
    order = sorted(range(1000), key=lambda i: sizes[i])
    ids = [order[int((k + 0.5) * 1000 / n)] for k in range(n)]
    rows = []
    for i in ids:
        g = G.corpus_app(i)
        app = gd.load(g, stream=torch.cuda.current_stream().cuda_stream)
        st = app.build()
        ptr, pairs = app.read_all_facts(0)
        P, Q, W = layout_sizes(g)
        n_m = np.bincount(g.node_method, minlength=len(P))
        cell = int((P * Q * ((n_m + 63) // 64) * 8).sum())
        node = np.repeat(np.arange(g.n_nodes), np.diff(ptr.astype(np.int64)))
        slot = (pairs >> np.uint64(32)).astype(np.int64)
        nz_rows = len(np.unique(node.astype(np.int64) * (1 << 32) + slot)) if len(pairs) else 0
        Wn = W[g.node_method]
        # stored rows weighted by their method's W: count rows per node, then weight
        uniq = np.unique(node.astype(np.int64) * (1 << 32) + slot) if len(pairs) else np.zeros(0, np.int64)
        row_words = int(Wn[(uniq >> 32)].sum()) if len(uniq) else 0
        sparse = 8 * g.n_nodes + 4 * nz_rows + 8 * row_words
        rows.append({"app": i, "nodes": g.n_nodes, "pairs": int(len(pairs)), "node_major": int(st["fact_bytes"]),
                     "cell_major": cell, "row_sparse": int(sparse), "set_tight": 8 * int(len(pairs))})
        r = rows[-1]
        print(f"app {i:4d} nodes {g.n_nodes:8d}  node-major {r['node_major'] / 1e6:8.1f} MB  cell-major "
              f"{cell / 1e6:8.1f} MB  row-sparse {sparse / 1e6:7.1f} MB  set {r['set_tight'] / 1e6:7.1f} MB", flush=True)
        app.free()
    for k in ("cell_major", "row_sparse", "set_tight"):
        v = [r[k] / r["node_major"] for r in rows]
        print(f"{k:>11} / node-major: mean {np.mean(v):.3f}  min {np.min(v):.3f}  max {np.max(v):.3f}")
    if out:
        json.dump({"what": "fact-store footprint of MAT layout variants (scripts/footprint.py)", "apps": rows},
                  open(out, "w"), indent=1)


if __name__ == "__main__":
    main()
