"""GPU tests of the corpus path that bench.py times (paper_conf_ipps_yuwobby20_b200/corpus.py):
released fact stores (gdroid_release_facts / build_opts.release_facts), the device-resident
shard with asynchronous builds, and the end-to-end pipeline's fact readback (Alg. 3 l.17
h_fact <- d_fact) compared with the oracle pair for pair."""
from __future__ import annotations

import numpy as np
import pytest

import oracle
import paper_conf_ipps_yuwobby20_b200 as gd
from paper_conf_ipps_yuwobby20_b200 import corpus
from synth import generator as G
from synth import random_tiny

pytestmark = pytest.mark.gpu


def test_release_facts_keeps_digests_and_rebuilds():
    gs = [random_tiny(s, wide_pad=(90 if s % 2 else 0)) for s in range(300, 340)]
    app = gd.load(gs)
    app.build(release_facts=True)
    digs = app.app_digests().copy()
    for k in (0, 7):
        per, dk = app.node_digests(k)
        assert dk == int(digs[k])
    with pytest.raises(gd.GdroidError) as e:         # facts are gone until the next build
        app.read_facts(0)
    assert e.value.code == -5
    app.release_facts()                              # idempotent
    app.build()                                      # re-allocates the store
    assert np.array_equal(app.app_digests(), digs)
    for k, g in enumerate(gs):
        r = oracle.build_idfg(g)
        ptr, pairs = app.read_all_facts(k)
        assert np.array_equal(ptr, r.ptr) and np.array_equal(pairs, r.pairs), g.name
        assert int(digs[k]) == r.app_digest
    app.release_facts()
    with pytest.raises(gd.GdroidError):
        app.read_all_facts(0)
    app.free()


def test_device_shard_async_steps_match_oracle():
    """Several batches, all tables resident, builds enqueued asynchronously back to back on
    one stream with released fact stores: every app equals the oracle (digest + per node)."""
    gs = {i: random_tiny(2000 + i, max_stmts=6, wide_pad=(120 if i % 5 == 0 else 0)) for i in range(60)}
    batches = [list(range(b, min(60, b + 13))) for b in range(0, 60, 13)]
    sh = corpus.DeviceShard(batches, gs)
    res = corpus.run_rank(sh, steps=2, warmup=1, barrier=lambda: None, timer=lambda fn: (fn(), 1.0)[1])
    for b, h in zip(batches, sh.handles):
        for k, i in enumerate(b):
            r = oracle.build_idfg(gs[i])
            assert res.digests[i] == r.app_digest
            per, _ = h.node_digests(k)
            assert np.array_equal(per, r.node_digest)
    assert all(s["alg_bytes"] > 0 for s in res.counted)
    sh.free()


def test_pipelined_fact_readback_equals_oracle():
    """run_pipelined (loader thread + pinned readback buffers) on small corpus apps: the read
    back IDFG equals the oracle's pair for pair."""
    ids = [4, 8, 5]                                  # 34K / 31K / 44K nodes
    apps = {i: G.corpus_app(i) for i in ids}
    seen = {}

    def on_facts(i, ptr, pairs):
        seen[i] = (ptr.copy(), pairs.copy())

    out = corpus.run_pipelined([[4, 8], [5]], lambda i: apps[i], readback="facts", on_facts=on_facts)
    assert sorted(seen) == sorted(ids)
    assert sum(br.d2h_bytes for br in out) > 8 * sum(apps[i].n_nodes for i in ids)
    for i in ids:
        r = oracle.build_idfg(apps[i])
        ptr, pairs = seen[i]
        assert np.array_equal(ptr, r.ptr) and np.array_equal(pairs, r.pairs), f"corpus{i}"


def test_pipelined_loader_error_surfaces():
    """A load failure in the loader thread is re-raised in the consumer (no hang)."""
    bad = random_tiny(1)
    bad.module_insts = bad.module_insts.copy()
    bad.module_insts[:] = 0                          # pools lose their sites: V1 fails (E_POOL)
    with pytest.raises(gd.GdroidError):
        corpus.run_pipelined([[0], [1]], lambda i: random_tiny(5) if i == 0 else bad)


def test_async_batch_readback_and_reserve_sms():
    """gdroid_read_batch_facts_async into pinned buffers equals the synchronous readback; a
    too-small pairs buffer is reported (nothing copied); a build with reserve_sms (smaller
    persistent grid) reaches the same fixed point."""
    gs = [random_tiny(s, wide_pad=(90 if s % 3 == 0 else 0)) for s in range(500, 560)]
    app = gd.load(gs)
    app.build()
    digs = app.app_digests().copy()
    ptr, pairs = app.read_batch_facts()
    bufs = corpus.ReadbackBuffers()
    n = sum(app.n_nodes)
    assert app.read_batch_facts_async(bufs.ptr.get(n + 1), bufs.pairs.get(max(1, len(pairs) - 1)),
                                      bufs.total.get(1)) is False
    assert app.read_batch_facts_async(bufs.ptr.get(n + 1), bufs.pairs.get(len(pairs) + 8), bufs.total.get(1))
    app.stream_sync()
    assert int(bufs.total.get(1)[0]) == len(pairs)
    assert np.array_equal(bufs.ptr.get(n + 1), ptr)
    assert np.array_equal(bufs.pairs.get(len(pairs)), pairs)
    app.build(reserve_sms=16)
    assert np.array_equal(app.app_digests(), digs)
    app.free()
