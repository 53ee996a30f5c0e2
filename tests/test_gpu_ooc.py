"""Out-of-core sub-graph streaming (ooc.py) and the
incremental-build API under it (keep_facts, gdroid_stage_seeds, import/export) on the GPU: the
sub-graph iteration reaches the same least fixed point as the oracle, pair for pair."""
from __future__ import annotations

import numpy as np
import pytest

import oracle
import paper_conf_ipps_yuwobby20_b200 as gd
from paper_conf_ipps_yuwobby20_b200 import ooc
from synth import generator as G
from synth import random_tiny

pytestmark = pytest.mark.gpu


def _same(ptr, pairs, r, label):
    assert np.array_equal(ptr, r.ptr) and np.array_equal(pairs, r.pairs), label


@pytest.mark.parametrize("seed", range(24))
def test_ooc_random_tiny(seed):
    g = random_tiny(3000 + seed, n_methods=3, max_stmts=6, wide_pad=(100 if seed % 3 == 0 else 0))
    o = ooc.OutOfCore(g, 1 + seed % 3)
    o.run()
    _same(*o.read_all_facts(), oracle.build_idfg(g), g.name)
    o.free()


@pytest.mark.parametrize("name,K", [("small", 4), ("median", 3)])
def test_ooc_presets(name, K):
    g = G.preset(name)
    o = ooc.OutOfCore(g, K)
    st = o.run()
    assert st.sweeps >= 2 and st.seeds > 0
    assert st.peak_resident_fact_bytes <= 2 * max(h.fact_bytes for h in o.handles)
    _same(*o.read_all_facts(), oracle.build_idfg(g), name)
    o.free()


def test_incremental_build_equals_fresh():
    """keep_facts: export the facts of a finished build, import them into a released store and
    rebuild incrementally with no seeds -> unchanged; staged seeds outside the pools -> E_POOL."""
    gs = [random_tiny(s, wide_pad=(70 if s % 2 else 0)) for s in range(400, 430)]
    app = gd.load(gs)
    app.build()
    digs = app.app_digests().copy()
    host = np.zeros(app.fact_bytes // 8, dtype=np.uint64)
    app.export_facts(host)
    app.stream_sync()
    app.release_facts()
    app.import_facts(host)
    st = app.build(keep_facts=True)
    assert np.array_equal(app.app_digests(), digs) and st["node_visits"] == 0
    app.stage_seeds(np.array([0], np.uint32), np.array([0, 1], np.uint64),
                    np.array([(0xFFFFFFF0 << 32) | 0], np.uint64))
    with pytest.raises(gd.GdroidError) as e:
        app.build(keep_facts=True)
    assert e.value.code == -2
    app.free()
