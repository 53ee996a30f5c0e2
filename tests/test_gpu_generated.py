"""GPU parity on the generated configs (BASELINE.json configs[1..3]): every node's fact set
equals the oracle's (small, median: full pair comparison; digests for all)."""
from __future__ import annotations

import numpy as np
import pytest

import oracle
import paper_conf_ipps_yuwobby20_b200 as gd
from synth import generator as G

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("name", ["small", "median"])
def test_preset_full_parity(name):
    g = G.preset(name)
    r = oracle.build_idfg(g)
    app = gd.load(g)
    st = app.build()
    ptr, pairs = app.read_all_facts(0)
    assert np.array_equal(ptr, r.ptr), "per-node fact counts differ"
    assert np.array_equal(pairs, r.pairs)
    per, dig = app.node_digests()
    assert np.array_equal(per, r.node_digest) and dig == r.app_digest
    assert st["node_visits"] > 0 and st["rounds"] > 0


def test_small_seeds_batch():
    """Eight small apps with other seeds, batched in one handle (shared rounds)."""
    gs = [G.preset("small", seed=s) for s in range(100, 108)]
    app = gd.load(gs)
    app.build()
    d = app.app_digests()
    for k, g in enumerate(gs):
        assert int(d[k]) == oracle.build_idfg(g).app_digest, g.name
