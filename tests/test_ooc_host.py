"""Host side of the out-of-core sub-graph split (paper_conf_ipps_yuwobby20_b200/ooc.py;
SURVEY §8(f)4): partition + sub-graph construction, checked on CPU.  Every
node is owned by exactly one sub-graph, every crossing edge ends in a proxy of its target,
and every sub-graph passes the library's input validation (V1-V6) — on a host without a GPU
the load then stops at the device upload, never at validation."""
from __future__ import annotations

import numpy as np
import pytest

import paper_conf_ipps_yuwobby20_b200 as gd
from paper_conf_ipps_yuwobby20_b200 import ooc
from synth import generator as G
from synth import random_tiny


def _check_split(g, K):
    part = ooc.partition_methods(g, K)
    subs = [ooc.make_subgraph(g, part, k) for k in range(K)]
    N = len(g.node_kind)
    owner = np.zeros(N, dtype=np.int64)
    for sg in subs:
        owner[sg.glob[sg.owned]] += 1
    assert (owner == 1).all()
    rp = g.row_ptr.astype(np.int64)
    src = np.repeat(np.arange(N), np.diff(rp))
    cross = part[g.node_method[src]] != part[g.node_method[g.col]]
    assert set(np.unique(g.edge_kind[cross]).tolist()) <= {ooc.E_CALL, ooc.E_RET}
    for e in np.nonzero(cross)[0][:2000]:
        k = part[g.node_method[src[e]]]
        assert int(g.col[e]) in set(subs[k].proxy_glob.tolist())
    for sg in subs:
        try:
            gd.load(sg.icfg)
        except gd.GdroidError as ex:
            assert ex.code not in (-1, -2), str(ex)      # not an input (validation) error
    return subs


@pytest.mark.parametrize("seed", range(40))
def test_split_random_tiny(seed):
    g = random_tiny(seed, n_methods=3, max_stmts=6)
    _check_split(g, 1 + seed % 3)


def test_split_small_preset():
    g = G.preset("small")
    subs = _check_split(g, 4)
    assert sum(len(s.proxies) for s in subs) > 0
