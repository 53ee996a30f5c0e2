"""GPU parity: the CUDA path (through the C ABI) vs the CPU oracle, bit-exact per node.

Exactly one result is correct (the least fixed point is unique, DESIGN.md §3 C4), so every
node's fact set must equal the oracle's pair for pair; digests must match too.
"""
from __future__ import annotations

import numpy as np
import pytest

import oracle
import paper_conf_ipps_yuwobby20_b200 as gd
from programs import fig2, load_expected, tiny, tiny2, tiny_args
from synth import random_tiny
from synth.reductions import random_inline_pair, random_rd, random_ssa_loop

pytestmark = pytest.mark.gpu


def _assert_same(app, k, g, r, label=""):
    ptr, pairs = app.read_all_facts(k)
    if not (np.array_equal(ptr, r.ptr) and np.array_equal(pairs, r.pairs)):
        for n in range(g.n_nodes):
            a = set(pairs[ptr[n]:ptr[n + 1]].tolist())
            b = set(r.facts(n).tolist())
            assert a == b, f"{label} node {n}: gpu-only {sorted(a - b)[:8]} oracle-only {sorted(b - a)[:8]}"
        raise AssertionError(f"{label}: CSR layout differs")


@pytest.mark.parametrize("which", ["tiny", "tiny_m2", "tiny2", "fig2", "tiny_args", "tiny_args_wide"])
def test_golden_programs(which):
    if which == "fig2":
        g = fig2()[0]
    elif which == "tiny2":
        g, L, slots, insts = tiny2()
    elif which.startswith("tiny_args"):      # 5-param call, one local passed 3 times (narrow / |Q|>64)
        g, L, slots, insts = tiny_args(wide_pad=(100 if which.endswith("wide") else 0))
    else:
        g, L, slots, insts = tiny(m2_entry=(which == "tiny_m2"))
    app = gd.load(g)
    st = app.build()
    r = oracle.build_idfg(g)
    _assert_same(app, 0, g, r, which)
    per, dig = app.node_digests()
    assert dig == r.app_digest and np.array_equal(per, r.node_digest)
    assert st["rounds"] > 0 and st["node_visits"] > 0
    if which != "fig2":      # and against the hand-computed fixture directly
        exp = load_expected("tiny_args" if which.startswith("tiny_args") else which)
        inv_s = {v: k for k, v in slots.items()}
        inv_i = {v: k for k, v in insts.items()}
        for lab, n in L.items():
            got = {(inv_s[int(p) >> 32], inv_i[int(p) & 0xFFFFFFFF]) for p in app.read_facts(n)}
            assert got == exp[lab], lab


@pytest.mark.parametrize("chunk", range(4))
def test_random_tiny_batches(chunk):
    """600 seeded random tiny ICFGs (every node/edge kind, recursion, projection), batched
    into one handle (shared device rounds), each compared with its own oracle run."""
    seeds = range(chunk * 150, chunk * 150 + 150)
    gs = [random_tiny(s) for s in seeds]
    app = gd.load(gs)
    app.build()
    digs = app.app_digests()
    for k, g in enumerate(gs):
        r = oracle.build_idfg(g)
        _assert_same(app, k, g, r, g.name)
        assert int(digs[k]) == r.app_digest


def test_reduction_programs_batch():
    gs = [random_rd(s) for s in range(100)] + [random_ssa_loop(s)[0] for s in range(100)]
    for s in range(60):
        P, Q, _, _ = random_inline_pair(s)
        gs += [P, Q]
    app = gd.load(gs)
    app.build()
    for k, g in enumerate(gs):
        _assert_same(app, k, g, oracle.build_idfg(g), g.name)


def test_loop_modes_and_rebuild_identical():
    gs = [random_tiny(s, max_stmts=7) for s in range(1000, 1100)]
    app = gd.load(gs)
    s0 = app.build(loop_mode=0)
    d0 = app.app_digests().copy()
    s1 = app.build(loop_mode=1)
    d1 = app.app_digests().copy()
    s2 = app.build(loop_mode=0, blocks=3)      # few CTAs: many nodes per warp per round
    d2 = app.app_digests().copy()
    assert np.array_equal(d0, d1) and np.array_equal(d0, d2)
    assert s1["kernel_launches"] > s0["kernel_launches"]
    for k in (0, 17, 99):
        _assert_same(app, k, gs[k], oracle.build_idfg(gs[k]))


def test_async_build_and_errors():
    g = tiny()[0]
    app = gd.load(g)
    with pytest.raises(gd.GdroidError) as e:
        app.read_facts(0)                    # before any build
    assert e.value.code == -5
    assert app.build(asynchronous=True) is None
    with pytest.raises(gd.GdroidError):
        app.build()                          # still pending
    st = app.sync()
    assert st["rounds"] > 0
    with pytest.raises(gd.GdroidError) as e:
        app.read_facts(g.n_nodes)
    assert e.value.code == -6
    with pytest.raises(gd.GdroidError) as e:
        app.build(max_rounds=2)
    assert e.value.code == -8


def test_empty_and_degenerate():
    """Degenerate inputs: a method whose entry has no successor; an app whose only entry
    reaches nothing; unreachable methods (A5) keep empty sets."""
    from synth import IcfgBuilder
    b = IcfgBuilder(n_fields=1)
    d = b.add_module()
    m = b.add_method(d, 0, 1)           # entry and exit, no edge between them
    b.add_entry(m)
    g = b.build()
    app = gd.load(g)
    app.build()
    ptr, pairs = app.read_all_facts(0)
    assert len(pairs) == 0
    r = oracle.build_idfg(g)
    assert r.app_digest == app.node_digests()[1] == 0


@pytest.mark.parametrize("pad", [70, 150, 300])
def test_wide_pool_batches(pad):
    """Pools of > 64 instances (W = 2/4/8 words per row): the row-occupancy path, with the real
    sites straddling word boundaries, against the oracle on 120 random tiny ICFGs."""
    gs = [random_tiny(s, wide_pad=pad) for s in range(5000 + pad, 5120 + pad)]
    app = gd.load(gs)
    app.build()
    digs = app.app_digests()
    for k, g in enumerate(gs):
        r = oracle.build_idfg(g)
        _assert_same(app, k, g, r, g.name)
        assert int(digs[k]) == r.app_digest
    app.build(loop_mode=1)                       # same results through per-round launches
    assert np.array_equal(app.app_digests(), digs)


def test_wide_and_narrow_mixed_batch():
    """Wide and narrow apps in one handle (the wide instantiation serves both layouts)."""
    gs = [random_tiny(s, wide_pad=(100 if s % 2 else 0)) for s in range(7000, 7060)]
    app = gd.load(gs)
    app.build()
    for k, g in enumerate(gs):
        _assert_same(app, k, g, oracle.build_idfg(g), g.name)


@pytest.mark.parametrize("variant", ["mat", "mat_grp", "gdroid"])
@pytest.mark.parametrize("blocks", [0, 3])
def test_ablation_variants(variant, blocks):
    """The ablation schedules (MAT / MAT+GRP / MAT+GRP+MER) reach the same
    least fixed point: narrow and wide random tiny ICFGs in one handle; with 3 CTAs (24 warps)
    most rounds exceed one wave, so MER's head/tail split defers tails."""
    gs = [random_tiny(s, wide_pad=(90 if s % 3 == 0 else 0)) for s in range(9000, 9120)]
    app = gd.load(gs)
    st = app.build(variant=variant, blocks=blocks)
    digs = app.app_digests()
    for k, g in enumerate(gs):
        r = oracle.build_idfg(g)
        _assert_same(app, k, g, r, f"{variant}/{g.name}")
        assert int(digs[k]) == r.app_digest
    assert st["rounds"] > 0


@pytest.mark.parametrize("which", ["tiny", "tiny_m2", "tiny2", "fig2"])
def test_plain_variant_golden(which):
    """PLAIN (set-based, thread per node; Alg. 2) on the hand-written programs."""
    g = fig2()[0] if which == "fig2" else (tiny2()[0] if which == "tiny2" else tiny(m2_entry=(which == "tiny_m2"))[0])
    app = gd.load(g, plain=True)
    st = app.build(variant="plain")
    r = oracle.build_idfg(g)
    _assert_same(app, 0, g, r, f"plain/{which}")
    per, dig = app.node_digests()
    assert dig == r.app_digest and np.array_equal(per, r.node_digest)
    assert st["node_visits"] > 0 and st["fact_bytes"] > 0
    app.build()                                   # the same handle runs the MAT path too
    _assert_same(app, 0, g, r, f"mat-after-plain/{which}")


@pytest.mark.parametrize("chunk", range(2))
def test_plain_variant_random(chunk):
    """PLAIN on 80 random tiny ICFGs (narrow and wide pools; every node/edge kind, recursion,
    projection) — one handle each, as the plain variant takes one app."""
    for s in range(11000 + chunk * 40, 11040 + chunk * 40):
        g = random_tiny(s, wide_pad=(80 if s % 4 == 0 else 0))
        app = gd.load(g, plain=True)
        app.build(variant="plain")
        r = oracle.build_idfg(g)
        _assert_same(app, 0, g, r, f"plain/{g.name}")
        assert app.node_digests()[1] == r.app_digest
        app.free()


def test_plain_variant_errors():
    g = tiny()[0]
    app = gd.load(g)                              # not loaded for PLAIN
    with pytest.raises(gd.GdroidError) as e:
        app.build(variant="plain")
    assert e.value.code == -5
    with pytest.raises(ValueError):
        gd.load([g, g], plain=True)


@pytest.mark.parametrize("wide", [0, 90])
def test_uncounted_instantiation_same_results(wide):
    """no_byte_model=1 runs the kernel instantiation without the byte-model counters: same
    fixed point (oracle), visits still counted, byte models reported as 0."""
    gs = [random_tiny(s, wide_pad=wide) for s in range(12000, 12080)]
    app = gd.load(gs)
    st = app.build(byte_model=False)
    assert st["alg_bytes"] == 0 and st["dense_bytes"] == 0 and st["node_visits"] > 0
    for k, g in enumerate(gs):
        _assert_same(app, k, g, oracle.build_idfg(g), g.name)
    st1 = app.build(byte_model=True)
    assert st1["alg_bytes"] > 0 and st1["dense_bytes"] >= st1["alg_bytes"]
    app.build(byte_model=False, loop_mode=1)
    for k in (0, 41, 79):
        _assert_same(app, k, gs[k], oracle.build_idfg(gs[k]))


def test_loader_sorted_key_paths(monkeypatch):
    """The loader's fallback for apps with too many modules / fields for the dense (module, field)
    and (module, module) mark tables (GDROID_LOADER_SPARSE forces it): same tables, same facts."""
    monkeypatch.setenv("GDROID_LOADER_SPARSE", "1")
    gs = [random_tiny(s) for s in range(900, 960)] + [tiny2()[0]]
    app = gd.load(gs)
    app.build()
    digs = app.app_digests()
    for k, g in enumerate(gs):
        r = oracle.build_idfg(g)
        _assert_same(app, k, g, r, g.name)
        assert int(digs[k]) == r.app_digest


def test_hybrid_schedule_limits_and_async():
    """Large narrow batches run the hybrid light/heavy launches: a round limit
    still stops the build (GDROID_E_LIMIT), an async build completes through gdroid_sync, a
    small grid gives the same fixed point, and every run matches the stored oracle digest."""
    import json
    import os
    from synth import generator as G
    fx = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "oracle_digests.json")))
    g = G.preset("median")
    app = gd.load(g)
    with pytest.raises(gd.GdroidError) as e:
        app.build(max_rounds=5)
    assert e.value.code == -8
    assert app.build(asynchronous=True) is None
    st = app.sync()
    assert st["rounds"] > 0 and st["kernel_launches"] >= 3
    assert str(int(app.app_digests()[0])) == fx["median"]["app_digest"]
    app.build(blocks=37)
    assert str(int(app.app_digests()[0])) == fx["median"]["app_digest"]
    app.free()


@pytest.mark.parametrize("chunk", range(2))
def test_cell_major_variant_random(chunk):
    """CELL: the paper's cell-major per-method matrices (Fig. 5b)
    as the fact store of the thread-per-node schedule, on 60 random tiny ICFGs (narrow and wide
    pools, arity up to 5) and the hand goldens — pair for pair against the oracle."""
    gs = [random_tiny(s, wide_pad=(80 if s % 4 == 0 else 0)) for s in range(13000 + chunk * 30, 13030 + chunk * 30)]
    if chunk == 0:
        gs += [tiny(m2_entry=True)[0], tiny2()[0], fig2()[0], tiny_args()[0], tiny_args(100)[0]]
    for g in gs:
        app = gd.load(g, plain=True)
        st = app.build(variant="cell")
        r = oracle.build_idfg(g)
        _assert_same(app, 0, g, r, f"cell/{g.name}")
        per, dig = app.node_digests()
        assert dig == r.app_digest and np.array_equal(per, r.node_digest)
        assert st["fact_bytes"] > 0
        app.free()


@pytest.mark.parametrize("blocks", [0, 2])
def test_sbda_schedule(blocks):
    """SBDA (SURVEY §8(f)3 as a schedule, DESIGN.md §5.6 / reading R8): one CTA per method per
    pass with shared-memory local worklists; narrow + wide random tiny ICFGs (arity up to 5,
    recursion, projection) and the goldens in one batch, pair for pair against the oracle."""
    gs = [random_tiny(s, max_stmts=7, wide_pad=(90 if s % 3 == 0 else 0)) for s in range(14000, 14120)]
    gs += [tiny(m2_entry=True)[0], tiny2()[0], fig2()[0], tiny_args()[0], tiny_args(100)[0]]
    app = gd.load(gs)
    st = app.build(variant="sbda", blocks=blocks)
    digs = app.app_digests()
    for k, g in enumerate(gs):
        r = oracle.build_idfg(g)
        _assert_same(app, k, g, r, f"sbda/{g.name}")
        assert int(digs[k]) == r.app_digest
    assert st["rounds"] > 0 and st["node_visits"] > 0
    app.build(variant="sbda", byte_model=False)        # rebuild: claims / local stamps reset
    assert np.array_equal(app.app_digests(), digs)


def test_heavy_round_instantiation_random_batch():
    """A narrow batch big enough for the hybrid schedule's heavy rounds (>= 2^17 nodes; the
    4-CTA/SM instantiation with paired half-warp inline items): 12,000 random
    tiny ICFGs (every node kind, arity up to 5, recursion, projection) — every app digest and
    the complete pair lists of 150 of them against the oracle."""
    gs = [random_tiny(s, max_stmts=7) for s in range(100000, 112000)]
    assert sum(g.n_nodes for g in gs) >= (1 << 17)
    app = gd.load(gs)
    st = app.build()
    assert st["kernel_launches"] >= 3                # the hybrid sequence ran
    digs = app.app_digests()
    for k, g in enumerate(gs):
        r = oracle.build_idfg(g)
        assert int(digs[k]) == r.app_digest, g.name
        if k % 80 == 0:
            _assert_same(app, k, g, r, g.name)
