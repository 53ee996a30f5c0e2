#!/usr/bin/env python3
"""Write tests/golden/corpus_digests.json: oracle results (ONLY oracle/ computes them) for every
app of the seeded 1000-app corpus (BASELINE.json configs[4]) except the clipped tail that uses
the worst-case shape (|Q| = 256: ~800 s of oracle each; covered by the `worst` preset entry of
oracle_digests.json).  Per app: generator version, node count, app digest and the
order-sensitive hash of the per-node digest array.  Runs the oracle in a process pool.
usage: make_corpus_digests.py [n_apps=1000] [procs=nproc]
       make_corpus_digests.py --wide [procs=4]   (then: the worst-shaped apps, merged in)
"""
import json
import os
import sys
import time
from multiprocessing import Pool

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "scripts"))
OUT = os.path.join(ROOT, "tests", "golden", "corpus_digests.json")


def one(i):
    import oracle
    from synth import generator as G
    from make_oracle_digests import node_hash
    g = G.corpus_app(i)
    r = oracle.build_idfg(g)
    e = {"n_nodes": g.n_nodes, "app_digest": str(r.app_digest),
         "node_digest_hash": str(node_hash(r.node_digest)), "oracle_s": round(r.seconds, 3)}
    if G.corpus_config(i).q_cap > 64:
        e["wide"] = True
    return i, e


def main_wide(procs):
    """--wide [procs]: add the worst-shaped apps (|Q| = 256, ~800 s of one core each) to the
    existing file (same generator version), one oracle process per app."""
    from synth import generator as G
    out = json.load(open(OUT))
    assert out["gen_version"] == G.GEN_VERSION, "narrow apps first"
    ids = [i for i in out.get("excluded_wide", []) if str(i) not in out["apps"]]
    t = time.time()
    with Pool(procs, maxtasksperchild=1) as p:
        for i, e in p.imap_unordered(one, ids):
            out["apps"][str(i)] = e
            out["excluded_wide"] = [j for j in out["excluded_wide"] if str(j) not in out["apps"]]
            out["apps"] = dict(sorted(out["apps"].items(), key=lambda kv: int(kv[0])))
            json.dump(out, open(OUT, "w"), indent=0)
            print(f"wide app {i}: {e['oracle_s']:.0f} s oracle, {time.time() - t:.0f} s", flush=True)


def main():
    from synth import generator as G
    if len(sys.argv) > 1 and sys.argv[1] == "--wide":
        return main_wide(int(sys.argv[2]) if len(sys.argv) > 2 else 4)
    n = int(sys.argv[1]) if len(sys.argv) > 1 else 1000
    procs = int(sys.argv[2]) if len(sys.argv) > 2 else os.cpu_count()
    ids = [i for i in range(n) if G.corpus_config(i).q_cap <= 64]
    t = time.time()
    out = {"gen_version": G.GEN_VERSION, "n_corpus": n,
           "excluded_wide": [i for i in range(n) if G.corpus_config(i).q_cap > 64], "apps": {}}
    sizes = G.corpus_sizes(n)
    with Pool(procs) as p:
        for k, (i, e) in enumerate(p.imap_unordered(one, sorted(ids, key=lambda i: -sizes[i]))):
            out["apps"][str(i)] = e
            if k % 50 == 0:
                print(f"{k}/{len(ids)} apps, {time.time() - t:.0f} s", flush=True)
    out["apps"] = dict(sorted(out["apps"].items(), key=lambda kv: int(kv[0])))
    json.dump(out, open(OUT, "w"), indent=0)
    print(f"wrote {len(out['apps'])} apps in {time.time() - t:.0f} s")


if __name__ == "__main__":
    main()
