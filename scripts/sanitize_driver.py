#!/usr/bin/env python3
"""Workload for compute-sanitizer (memcheck / racecheck / synccheck): the hot path on the hand
goldens, random tiny ICFGs (narrow and wide pools, arity up to 5), one incremental build with
staged seeds, and the small preset, each checked against the oracle.  No torch (plain CUDA
context of the library)."""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path[:0] = [ROOT, os.path.join(ROOT, "tests", "golden")]
import oracle  # noqa: E402
import paper_conf_ipps_yuwobby20_b200 as gd  # noqa: E402
from programs import tiny  # noqa: E402
from synth import generator as G  # noqa: E402
from synth import random_tiny  # noqa: E402

what = sys.argv[1] if len(sys.argv) > 1 else "all"
gs = [tiny(m2_entry=True)[0]] + [random_tiny(s, wide_pad=(100 if s % 3 == 0 else 0)) for s in range(48)]
app = gd.load(gs)
for variant in ("default", "mat", "gdroid"):
    app.build(variant=variant)
    for k, g in enumerate(gs):
        r = oracle.build_idfg(g)
        ptr, pairs = app.read_all_facts(k)
        assert np.array_equal(ptr, r.ptr) and np.array_equal(pairs, r.pairs), (variant, g.name)
host = np.zeros(app.fact_bytes // 8, dtype=np.uint64)
app.export_facts(host)
app.stream_sync()
app.release_facts()
app.import_facts(host)
app.build(keep_facts=True)
app.build(loop_mode=1)
app.free()
if what == "all":
    g = G.preset("small")
    a = gd.load(g)
    a.build()
    ref = oracle.build_idfg(g)
    assert a.node_digests()[1] == ref.app_digest
    a.free()
print("sanitize driver ok")
