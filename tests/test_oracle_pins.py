"""Pins of the CPU oracle against things other than itself (run with -m "not gpu").

Each test names what it pins and the passage / reading it follows.
"""
from __future__ import annotations

import numpy as np
import pytest

import oracle
from kleene import Sym, kleene, reach, to_sym
from reductions import andersen, reaching_definitions
from programs import tiny_args, fig2, load_expected, tiny, tiny2
from synth import random_tiny
from synth.reductions import random_inline_pair, random_rd, random_ssa_loop


def _named(g, slots, insts, r, n):
    inv_s = {v: k for k, v in slots.items()}
    inv_i = {v: k for k, v in insts.items()}
    return {(inv_s[s], inv_i[o]) for (s, o) in r.fact_set(n)}


# --------------------------------------------------------------------- golden, by hand
@pytest.mark.parametrize("variant", ["tiny", "tiny_m2"])
def test_golden_tiny(variant):
    """Hand-computed IN sets of the tiny config (BASELINE.json configs[0]); C2/C3 tables."""
    g, L, slots, insts = tiny(m2_entry=(variant == "tiny_m2"))
    assert g.n_nodes == 29 and g.n_methods == 3 and len(slots) <= 16 and len(insts) <= 16
    exp = load_expected(variant)
    assert set(exp) == set(L), "fixture must list every node"
    r = oracle.build_idfg(g)
    for lab, n in L.items():
        assert _named(g, slots, insts, r, n) == exp[lab], lab


def test_golden_tiny2_projection():
    """Hand-computed projection example (two modules, partial pools; C1/C3, A9)."""
    g, L, slots, insts = tiny2()
    exp = load_expected("tiny2")
    assert set(exp) == set(L)
    r = oracle.build_idfg(g)
    for lab, n in L.items():
        assert _named(g, slots, insts, r, n) == exp[lab], lab


@pytest.mark.parametrize("pad", [0, 100])
def test_golden_tiny_args(pad):
    """Hand-computed IN sets of a 5-parameter call with one local passed three times (C3 maps
    it to every such parameter), narrow and wide pools (padding never flows)."""
    g, L, slots, insts = tiny_args(wide_pad=pad)
    exp = load_expected("tiny_args")
    assert set(exp) == set(L)
    r = oracle.build_idfg(g)
    for lab, n in L.items():
        assert _named(g, slots, insts, r, n) == exp[lab], lab


# --------------------------------------------------------------------- the paper's figures
def test_fig2_round_sequence():
    """Fig. 2 worklist sequence {entry},{L1},{L2,L4},{L3,L5},{L6},{L7},{…,L1},{…,L2,L4}
     and the re-insertion of L1 after L7."""
    g, L = fig2()
    rounds = [set(r) for r in oracle.bsp_rounds(g)]
    nm = lambda *ls: {L[x] for x in ls}
    printed = [nm("entry"), nm("L1"), nm("L2", "L4"), nm("L3", "L5"), nm("L6"), nm("L7")]
    assert rounds[:6] == printed
    assert L["L1"] in rounds[6] and nm("L2", "L4") <= rounds[7]
    # our reading of the "…" placeholders: exit in round 7, nothing extra in 8
    assert rounds[6:] == [nm("exit", "L1"), nm("L2", "L4"), nm("L3", "L5"), nm("L6"), nm("L7")]
    r = oracle.build_idfg(g)
    x_o = {(0, 1)}
    for lab in ("L1", "L2", "L3", "L4", "L5", "L6", "L7", "exit"):
        assert r.fact_set(L[lab]) == x_o, lab       # fact(i)' after the revisit
    assert r.fact_set(L["entry"]) == set()


def test_fig7_merge():
    """Fig. 7: 36 sources, head N0..N31, tail N32..N35; the
    destinations contain N33 -> the next worklist holds N33 once."""
    wl = list(range(36))
    dests = [100, 101, 33, 102]
    head, nxt = oracle.mer_merge(wl, dests)
    assert head == 32
    assert sorted(nxt) == sorted({100, 101, 102, 32, 33, 34, 35})
    assert nxt.count(33) == 1 and len(nxt) == 7
    assert nxt[-4:] == [32, 33, 34, 35]             # printed order {Nx..Ny, N32..N35}
    h2, n2 = oracle.mer_merge(list(range(20)), [5, 5, 7])   # <= 32: whole list is head
    assert h2 == 20 and n2 == [5, 7]


# --------------------------------------------------------------------- brute force
@pytest.mark.parametrize("seed", range(400))
def test_kleene_equals_worklist(seed):
    """Least fixed point: the worklist oracle == Jacobi/Kleene iteration from ⊥ (C4)."""
    g = random_tiny(seed)
    r = oracle.build_idfg(g)
    S, K = kleene(g)
    for n in range(g.n_nodes):
        assert to_sym(S, r.facts(n)) == K[n], (seed, n)


@pytest.mark.parametrize("seed", range(200))
def test_order_independence_and_postfix(seed):
    """FIFO, LIFO and random orders give one IN; applying the transfer
    functions once more changes nothing (post-fixpoint); unreached nodes stay ∅ (A5)."""
    g = random_tiny(seed + 10_000, max_stmts=7)
    base = oracle.build_idfg(g, order=0)
    assert oracle.check_postfix(g, base) == 0
    for order, s in ((1, 0), (2, 1), (2, 2)):
        r = oracle.build_idfg(g, order=order, seed=s)
        assert np.array_equal(r.ptr, base.ptr) and np.array_equal(r.pairs, base.pairs)
    R = reach(g)
    for n in range(g.n_nodes):
        if n not in R:
            assert len(base.facts(n)) == 0


@pytest.mark.parametrize("seed", range(150))
def test_pool_containment(seed):
    """IN(n) ⊆ P_m × Q_m (C1): every stored fact lies in its method's pools."""
    g = random_tiny(seed + 20_000)
    S = Sym(g)
    r = oracle.build_idfg(g)
    for n in range(g.n_nodes):
        m = int(g.node_method[n])
        for (s, o) in to_sym(S, r.facts(n)):
            assert S.in_pool(m, s, o), (seed, n, s, o)


@pytest.mark.parametrize("seed", range(60))
def test_full_pools_equal_single_module(seed):
    """With complete pools the projection π is the identity: splitting the methods of one
    program over two modules must not change any fact (C1/C3)."""
    import copy
    g1 = random_tiny(seed + 30_000, n_methods=3, n_modules=1, full_pools=True)
    g2 = copy.deepcopy(g1)
    g2.method_module = (np.arange(g2.n_methods) % 2).astype(np.uint32)
    I, G = g1.n_instances, g1.n_statics
    g2.module_inst_ptr = np.array([0, I, 2 * I], dtype=np.uint64)
    g2.module_insts = np.concatenate([np.arange(I), np.arange(I)]).astype(np.uint32)
    g2.module_static_ptr = np.array([0, G, 2 * G], dtype=np.uint64)
    g2.module_statics = np.concatenate([np.arange(G), np.arange(G)]).astype(np.uint32)
    r1, r2 = oracle.build_idfg(g1), oracle.build_idfg(g2)
    assert np.array_equal(r1.pairs, r2.pairs) and np.array_equal(r1.ptr, r2.ptr)


# --------------------------------------------------------------------- textbook reductions
@pytest.mark.parametrize("seed", range(300))
def test_reaching_definitions_reduction(seed):
    """NEW/CONST/PRIM/NOP only: (v,o) ∈ IN(n) iff a definition of v with instance o reaches n
    (ALSU §9.2.4) — pins C2's kill/gen for the one-time-generation group."""
    g = random_rd(seed)
    r = oracle.build_idfg(g)
    S = Sym(g)
    rd = reaching_definitions(g)
    for n in range(g.n_nodes):
        got = to_sym(S, r.facts(n))
        assert got == rd.get(n, set()), (seed, n)


@pytest.mark.parametrize("seed", range(400))
def test_andersen_reduction(seed):
    """Single loop, every local defined once: IN(loop head) = Andersen's points-to solution —
    pins C2 for COPY/SLOAD/SSTORE (single-layer) and FLOAD/FSTORE/ALOAD/ASTORE (double-layer,
    PAPER.md:947-964), NEW/CONST/PRIM/RETV."""
    g, head, body = random_ssa_loop(seed)
    r = oracle.build_idfg(g)
    S = Sym(g)
    assert to_sym(S, r.facts(head)) == andersen(g), seed


@pytest.mark.parametrize("seed", range(300))
def test_inlining_law(seed):
    """One call site, non-recursive callee: CALL/C2R/RET edges (C3) == inlining the callee."""
    P, Q, pairs, info = random_inline_pair(seed)
    rP, rQ = oracle.build_idfg(P), oracle.build_idfg(Q)
    SP, SQ = Sym(P), Sym(Q)
    nl0 = info["nl0"]

    def q_map(slot):          # P_inl slot -> P slot names
        if slot[0] == "L":
            return ("L", 0, slot[2]) if slot[2] < nl0 else ("L", 1, slot[2] - nl0)
        return slot

    for n, (nq, side) in pairs.items():
        keep_m = 0 if side == "caller" else 1
        keep = lambda s: s[0] != "L" or s[1] == keep_m
        a = {p for p in to_sym(SP, rP.facts(n)) if keep(p[0])}
        b = {(q_map(s), o) for (s, o) in to_sym(SQ, rQ.facts(nq))}
        b = {p for p in b if keep(p[0])}
        assert a == b, (seed, n, side)


# --------------------------------------------------------------------- digest (C8)
def _mix64(z):
    M = (1 << 64) - 1
    z &= M
    z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & M
    z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & M
    return z ^ (z >> 31)


def test_mix64_known_values():
    """splitmix64 finaliser: z=1 value from the published splitmix64 sequence step
    (seed 0 -> state 0x9e3779b97f4a7c15 -> output 0xe220a8397b1dcdaf)."""
    assert _mix64(0x9E3779B97F4A7C15) == 0xE220A8397B1DCDAF


@pytest.mark.parametrize("seed", range(30))
def test_digest_definition(seed):
    g = random_tiny(seed + 40_000)
    r = oracle.build_idfg(g)
    M = (1 << 64) - 1
    app = 0
    for n in range(g.n_nodes):
        d = 0
        for p in r.facts(n):
            d = (d + _mix64(_mix64(n) ^ int(p))) & M
        assert d == int(r.node_digest[n])
        app = (app + d) & M
    assert app == r.app_digest


# --------------------------------------------------------------------- validation
def test_validation_rejects():
    g, L, slots, insts = tiny()
    bad = tiny()[0]
    bad.method_n_params = bad.method_n_params.copy(); bad.method_n_params[1] = 2
    bad.method_n_locals = bad.method_n_locals.copy()
    with pytest.raises(oracle.OracleError) as e:
        oracle.build_idfg(bad)
    assert e.value.code == -1
    bad2 = tiny()[0]
    bad2.module_insts = bad2.module_insts[bad2.module_insts != 3].copy()   # drop o3 from pool
    bad2.module_inst_ptr = np.array([0, len(bad2.module_insts)], dtype=np.uint64)
    with pytest.raises(oracle.OracleError) as e:
        oracle.build_idfg(bad2)
    assert e.value.code == -2   # V1: NEW site o3 outside the module pool


# --------------------------------------------------------------------- straight-line closed forms
def _straight(stmts_fn):
    """Build `entry -> s1 -> ... -> sk -> exit` in one method (locals a,b,v,x,y,z + RET)."""
    from synth import IcfgBuilder
    b = IcfgBuilder(n_fields=2)                    # 0 = ARR, 1 = f
    TA = b.add_type([1]); TN = b.add_type([])
    o1 = b.add_instance(TA); o2 = b.add_instance(TA); o3 = b.add_instance(TA)
    o4 = b.add_instance(TN)
    d = b.add_module(insts=[o1, o2, o3, o4])
    m = b.add_method(d, 0, 7)
    V = {n: b.L(m, i) for i, n in enumerate("abvxyz")}
    body = stmts_fn(b, m, V, (o1, o2, o3, o4))
    b.chain(b.entry(m), *body, b.exit(m))
    b.add_entry(m)
    g = b.build()
    names = {i: n for i, n in enumerate("abvxyz")}
    names[6] = "R"
    return g, int(g.method_exit[0]), names


STRAIGHT = {
    # RETV kills RET_m: only the last return value survives (C2 RETV row)
    "retv_kill": (lambda b, m, V, o: [b.new(m, V["a"], o[0]), b.new(m, V["b"], o[1]),
                                      b.retv(m, V["a"]), b.retv(m, V["b"])],
                  {("a", 1), ("b", 2), ("R", 2)}),
    # heap updates are weak (A8): both stores to o1.f survive; load sees both
    "weak_heap": (lambda b, m, V, o: [b.new(m, V["x"], o[0]), b.new(m, V["y"], o[1]),
                                      b.fstore(m, V["x"], 1, V["y"]), b.new(m, V["z"], o[2]),
                                      b.fstore(m, V["x"], 1, V["z"]), b.fload(m, V["v"], V["x"], 1)],
                  {("x", 1), ("y", 2), ("z", 3), ("o1.f", 2), ("o1.f", 3), ("v", 2), ("v", 3)}),
    # v = v.f: GEN on X before the kill (C2 note)
    "self_load": (lambda b, m, V, o: [b.new(m, V["x"], o[0]), b.new(m, V["y"], o[1]),
                                      b.fstore(m, V["x"], 1, V["y"]), b.fload(m, V["x"], V["x"], 1)],
                  {("x", 2), ("y", 2), ("o1.f", 2)}),
    # v.f = v
    "self_store": (lambda b, m, V, o: [b.new(m, V["x"], o[0]), b.fstore(m, V["x"], 1, V["x"])],
                   {("x", 1), ("o1.f", 1)}),
    # load through NULL generates nothing but still kills v (A23)
    "null_load": (lambda b, m, V, o: [b.new(m, V["v"], o[0]), b.const(m, V["x"], 0),
                                      b.fload(m, V["v"], V["x"], 1)],
                  {("x", 0)}),
    # field not declared by the type: store and load generate nothing (C1: no heap slot)
    "no_field": (lambda b, m, V, o: [b.new(m, V["x"], o[3]), b.new(m, V["y"], o[0]),
                                     b.fstore(m, V["x"], 1, V["y"]), b.fload(m, V["v"], V["x"], 1)],
                 {("x", 4), ("y", 1)}),
    # arrays use the ARR pseudo-field only (C2 ALOAD/ASTORE = FLOAD/FSTORE with f = ARR)
    "arr_vs_field": (lambda b, m, V, o: [b.new(m, V["x"], o[0]), b.new(m, V["y"], o[1]),
                                         b.fstore(m, V["x"], 1, V["y"]), b.aload(m, V["v"], V["x"])],
                     {("x", 1), ("y", 2), ("o1.f", 2)}),
}


@pytest.mark.parametrize("case", sorted(STRAIGHT))
def test_straight_line_closed_forms(case):
    """Straight-line code: IN(exit) = f_k∘…∘f_1(∅), values derived by hand (C7)."""
    fn, expected = STRAIGHT[case]
    g, ex, names = _straight(fn)
    r = oracle.build_idfg(g)
    Lt = int(g.method_n_locals.sum())
    heap = {Lt + g.n_statics + i: f"o{i + 1}.f" for i in range(3)}   # o1..o3 have field f
    got = {(names.get(s, heap.get(s)), o) for (s, o) in r.fact_set(ex)}
    assert got == expected


@pytest.mark.parametrize("seed", range(60))
def test_kleene_equals_worklist_wide_pools(seed):
    """Same brute-force pin with > 64-instance pools (the padding instances never get facts)."""
    g = random_tiny(seed + 50_000, wide_pad=130)
    r = oracle.build_idfg(g)
    S, K = kleene(g)
    for n in range(g.n_nodes):
        assert to_sym(S, r.facts(n)) == K[n], (seed, n)
