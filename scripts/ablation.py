#!/usr/bin/env python3
"""Ablation of the paper's optimisations on B200 (Figs. 8-12).

Each app of a seeded corpus sample is loaded once (gdroid_load_icfg_plain: MAT tables + the
set-based state) and built with every variant; the build time is the library's CUDA-event time
of one build (zeroing + fixed point + digests), median of --reps after one warm-up.  Every
variant's app digest must equal the default path's (same least fixed point).

Reported, per app and summarised like the paper's figures:
  Fig. 9   MAT vs PLAIN            speedup of the matrix store over the set-based plain kernel
  Fig. 10  memory footprint        set-based bytes (allocated arrays + descriptors) vs MAT bytes
  Fig. 11  MAT+GRP vs MAT          class-segmented worklists
  Fig. 12  MAT+GRP+MER vs MAT+GRP  head/tail merging
  Fig. 8   each vs PLAIN, and the B200 default path vs PLAIN
usage: python scripts/ablation.py [--apps 24] [--reps 3] [--out gpurun_out/ablation.json]
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

VARIANTS = ["plain", "mat", "mat_grp", "gdroid", "default", "cell"]


def sample_ids(n_apps, n_corpus=1000, max_nodes=None):
    """Stratified sample of the corpus by size: every (n_corpus / n_apps)-th app in size order."""
    from synth import generator as G
    sizes = G.corpus_sizes(n_corpus)
    order = sorted(range(n_corpus), key=lambda i: sizes[i])
    if max_nodes:
        order = [i for i in order if sizes[i] <= max_nodes]
    step = len(order) / n_apps
    return [order[int(k * step + step / 2)] for k in range(n_apps)], sizes


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--apps", type=int, default=24)
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("--max-nodes", type=int, default=700_000, help="skip larger apps (plain is slow)")
    ap.add_argument("--cell-max-nodes", type=int, default=150_000,
                    help="CELL (cell-major matrices, SURVEY §8(f)2) only on apps up to this size (a visit gathers |P_m| x |Q_m| cells)")
    ap.add_argument("--out", default=os.path.join(ROOT, "gpurun_out", "ablation.json"))
    args = ap.parse_args()

    import torch
    import paper_conf_ipps_yuwobby20_b200 as gd
    from synth import generator as G

    torch.cuda.set_device(0)
    stream = torch.cuda.current_stream().cuda_stream
    ids, sizes = sample_ids(args.apps, max_nodes=args.max_nodes)
    rows = []
    for i in ids:
        g = G.corpus_app(i)
        t0 = time.time()
        app = gd.load(g, stream=stream, plain=True)
        row = {"app": i, "nodes": g.n_nodes, "edges": int(g.n_edges)}
        ref = None
        for v in VARIANTS:
            if v == "cell" and g.n_nodes > args.cell_max_nodes:
                continue
            app.build(variant=v)                               # warm-up
            ts, st = [], None
            for _ in range(args.reps):
                st = app.build(variant=v)
                ts.append(st["build_ns"] / 1e6)
            dig = int(app.node_digests()[1])
            if v == "default":
                ref = dig
            row[v] = {"ms": statistics.median(ts), "rounds": st["rounds"], "visits": st["node_visits"],
                      "fact_bytes": st["fact_bytes"], "digest": str(dig)}
        for v in VARIANTS:
            if v in row:
                assert row[v]["digest"] == str(ref), f"app {i}: {v} digest differs from the default path"
        app.free()
        rows.append(row)
        print(f"app {i:4d} nodes {g.n_nodes:8d}  " + "  ".join(f"{v} {row[v]['ms']:9.2f}" for v in VARIANTS if v in row)
              + f"  ({time.time() - t0:.1f}s)", flush=True)

    def ratio(a, b):
        return [r[a]["ms"] / r[b]["ms"] for r in rows if a in r and b in r]

    def summ(x):
        x = sorted(x)
        return {"mean": statistics.mean(x), "median": statistics.median(x), "min": x[0], "max": x[-1],
                "frac_lt_1": sum(1 for v in x if v < 1) / len(x)}

    mem = [r["plain"]["fact_bytes"] / r["mat"]["fact_bytes"] for r in rows]
    out = {
        "what": "per-app build-time speedups (CUDA events, median of reps) on a stratified corpus sample",
        "apps": len(rows), "reps": args.reps, "device": torch.cuda.get_device_name(0),
        "fig9_mat_vs_plain": summ(ratio("plain", "mat")),
        "fig11_grp_vs_mat": summ(ratio("mat", "mat_grp")),
        "fig12_mer_vs_mat_grp": summ(ratio("mat_grp", "gdroid")),
        "fig8_gdroid_vs_plain": summ(ratio("plain", "gdroid")),
        "default_vs_plain": summ(ratio("plain", "default")),
        "default_vs_gdroid": summ(ratio("gdroid", "default")),
        "fig10_set_bytes_over_mat_bytes": summ(mem),
        "f2_mat_vs_cell": summ(ratio("cell", "mat")),
        "f2_cell_bytes_over_mat_bytes": summ([r["cell"]["fact_bytes"] / r["mat"]["fact_bytes"] for r in rows if "cell" in r]),
        "paper": {"mat_vs_plain_avg": 26.7, "grp_vs_mat_note": "<1.5x for 76.3% of apps, <1x for 15.5%",
                  "mer_vs_mat_grp_avg": 1.94, "gdroid_vs_plain_avg": 71.3, "mat_memory": "-75% on average",
                  "hardware": "NVIDIA Tesla P40 (PAPER.md:1090-1100)"},
        "rows": rows,
    }
    os.makedirs(os.path.dirname(args.out), exist_ok=True)
    with open(args.out, "w") as fh:
        json.dump(out, fh, indent=1)
    for k, v in out.items():
        if isinstance(v, dict) and "mean" in v:
            print(f"{k:34s} mean {v['mean']:8.2f}  median {v['median']:8.2f}  min {v['min']:8.2f}  max {v['max']:8.2f}")


if __name__ == "__main__":
    main()
