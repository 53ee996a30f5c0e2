"""Seeded program families for the oracle's textbook-reduction pins.

Input construction only.  Each family is shaped so that the method's result
reduces to an independently known textbook problem (the solvers for those live
in tests/reductions.py, never here):

* ``random_rd``       — one method, only NOP/PRIM/CONST/NEW nodes, arbitrary CFG
  with loops: IN(n) = reaching definitions (Aho-Lam-Sethi-Ullman §9.2.4).
* ``random_ssa_loop`` — one method whose body is a single loop, every local
  defined at most once: IN(loop head) = Andersen's inclusion-based points-to.
* ``random_inline_pair`` — a caller with ONE call site to a non-recursive
  callee, plus the same program with the callee inlined: context-insensitive
  CALL/RET/C2R with one call site must equal inlining.
"""
from __future__ import annotations

import random
from typing import Dict, List, Tuple

from .icfg import (ALOAD, ASTORE, COPY, CONST, FLOAD, FSTORE, NEW, NOP, PRIM, RETV,
                   SLOAD, SSTORE, E_INTRA, Icfg, IcfgBuilder)
from .tiny_random import random_tiny


def random_rd(seed: int) -> Icfg:
    return random_tiny(seed, n_methods=1, n_modules=1, max_stmts=8, full_pools=True,
                       kinds=[NOP, PRIM, CONST, NEW, CONST, NEW], allow_calls=False)


def _universe(rng, b: IcfgBuilder):
    types = [b.add_type(rng.sample(range(b.n_fields), rng.randint(1, b.n_fields)))
             for _ in range(rng.randint(1, 3))]
    for _ in range(rng.randint(0, 2)):
        b.add_static()
    return types


def _emit(rng, b, m, kind, loc_def, loc_use, types, sites):
    """One intra-procedural statement of `kind` in method m; returns its node."""
    nf = b.n_fields
    if kind in (SLOAD, SSTORE) and b.n_statics == 0:
        kind = COPY if loc_def is not None else NOP
    if kind == NOP:
        return b.nop(m)
    if kind == PRIM:
        return b.prim(m, loc_def())
    if kind == CONST:
        if rng.random() < 0.3:
            return b.const(m, loc_def(), 0)
        o = b.add_instance(rng.choice(types)); sites.append(o)
        return b.const(m, loc_def(), o)
    if kind == NEW:
        o = b.add_instance(rng.choice(types)); sites.append(o)
        return b.new(m, loc_def(), o)
    if kind == COPY:
        return b.copy(m, loc_def(), loc_use())
    if kind == SLOAD:
        return b.sload(m, loc_def(), b.S(rng.randrange(b.n_statics)))
    if kind == SSTORE:
        return b.sstore(m, b.S(rng.randrange(b.n_statics)), loc_use())
    if kind == FLOAD:
        return b.fload(m, loc_def(), loc_use(), rng.randrange(nf))
    if kind == FSTORE:
        return b.fstore(m, loc_use(), rng.randrange(nf), loc_use())
    if kind == ALOAD:
        return b.aload(m, loc_def(), loc_use())
    if kind == ASTORE:
        return b.astore(m, loc_use(), loc_use())
    raise AssertionError(kind)


def random_ssa_loop(seed: int) -> Tuple[Icfg, int, List[int]]:
    """Returns (icfg, loop_head_node, body_nodes).  Every local has <= 1 definition."""
    rng = random.Random(seed)
    b = IcfgBuilder(n_fields=rng.randint(1, 3))
    types = _universe(rng, b)
    d = b.add_module()
    nl = rng.randint(2, 6)                      # locals 0..nl-2 + RET
    m = b.add_method(d, 0, nl)
    undefined = list(range(nl - 1))
    rng.shuffle(undefined)
    sites: List[int] = []
    body: List[int] = []
    n_stmts = rng.randint(3, 10)
    defining = [NEW, CONST, COPY, SLOAD, FLOAD, ALOAD, PRIM, NEW]
    storing = [SSTORE, FSTORE, ASTORE, NOP]
    ret_defined = False
    for _ in range(n_stmts):
        use = lambda: b.L(m, rng.randrange(nl - 1))
        r = rng.random()
        if r < 0.1 and not ret_defined:
            body.append(b.retv(m, use())); ret_defined = True
        elif r < 0.6 and undefined:
            v = undefined.pop()
            body.append(_emit(rng, b, m, rng.choice(defining), lambda: b.L(m, v), use, types, sites))
        else:
            body.append(_emit(rng, b, m, rng.choice(storing), None, use, types, sites))
    b.chain(b.entry(m), *body)
    b.edge(body[-1], body[0])                   # the loop
    b.edge(body[-1], b.exit(m))
    b.set_module(d, insts=list(range(1, len(b.inst_type))), statics=list(range(b.n_statics)))
    b.add_entry(m)
    return b.build(name=f"ssa_loop_{seed}"), body[0], body


def random_inline_pair(seed: int):
    """Returns (P, P_inl, corr) where corr maps P node -> (P_inl node, 'caller'|'callee').

    P:      m0: entry -> A -> CALL lhs = m1(args) -> RETSITE -> B -> exit  (optional loop B->A)
            m1: entry -> C -> exit  (branches inside C; exit always reachable)
    P_inl:  m0': entry -> A -> NOP_call -> [COPY p_j = a_j | PRIM l_i: fresh frame]
            -> NOP_e -> C' -> NOP_x -> [COPY lhs = RET'] -> NOP_r -> B -> exit
    m0 has no RETV (its RET local is shared by nothing); m1's RET is m0''s last local.
    """
    rng = random.Random(seed)
    nf = rng.randint(1, 3)
    n_types = rng.randint(1, 3)
    type_fields = [rng.sample(range(nf), rng.randint(1, nf)) for _ in range(n_types)]
    n_stat = rng.randint(0, 2)
    nl0 = rng.randint(2, 4)       # includes (unused) RET0
    np1 = rng.choice((1, 1, 2, 2, 3, 4, 5, 6))   # arity up to 6 (> 3: the args-table path)
    nl1 = np1 + rng.randint(0, 2) + 1
    kinds0 = [NOP, PRIM, CONST, NEW, COPY, SLOAD, SSTORE, FLOAD, FSTORE, ALOAD, ASTORE]
    kinds1 = kinds0 + [RETV, RETV]
    A = [rng.choice(kinds0) for _ in range(rng.randint(1, 4))]
    Bk = [rng.choice(kinds0) for _ in range(rng.randint(1, 3))]
    Ck = [rng.choice(kinds1) for _ in range(rng.randint(1, 5))]
    c_branches = [(rng.random(), rng.random()) for _ in range(rng.randint(0, 2))]
    loop = rng.random() < 0.5
    has_lhs = rng.random() < 0.7
    stream_seed = rng.getrandbits(32)

    def make(inline: bool):
        r2 = random.Random(stream_seed)           # identical statement operands in both
        b = IcfgBuilder(n_fields=nf)
        types = [b.add_type(f) for f in type_fields]
        for _ in range(n_stat):
            b.add_static()
        d = b.add_module()
        sites: List[int] = []
        corr: Dict[str, int] = {}
        if inline:
            m0 = b.add_method(d, 0, nl0 + nl1)
            cal = lambda i: b.L(m0, i)
            cee = lambda i: b.L(m0, nl0 + i)
            m1 = m0
        else:
            m0 = b.add_method(d, 0, nl0)
            m1 = b.add_method(d, np1, nl1)
            cal = lambda i: b.L(m0, i)
            cee = lambda i: b.L(m1, i)
        u0 = lambda: cal(r2.randrange(nl0 - 1))
        u1 = lambda: cee(r2.randrange(nl1 - 1))
        a_nodes = [_emit(r2, b, m0, k, u0, u0, types, sites) for k in A]
        lhs_i = r2.randrange(nl0 - 1)
        if np1 >= 2 and r2.random() < 0.4:         # one caller local passed as several actuals
            rep = r2.randrange(nl0 - 1)
            args = [rep if r2.random() < 0.8 else -1 for _ in range(np1)]
        else:
            args = [r2.randrange(nl0 - 1) if r2.random() < 0.8 else -1 for _ in range(np1)]
        b_nodes = [_emit(r2, b, m0, k, u0, u0, types, sites) for k in Bk]
        c_nodes = []
        for k in Ck:
            if k == RETV:
                c_nodes.append(b.retv(m1, u1()))
            else:
                c_nodes.append(_emit(r2, b, m1, k, u1, u1, types, sites))
        for i, n in enumerate(a_nodes): corr[f"A{i}"] = n
        for i, n in enumerate(b_nodes): corr[f"B{i}"] = n
        for i, n in enumerate(c_nodes): corr[f"C{i}"] = n
        lhs = cal(lhs_i) if has_lhs else None
        if inline:
            n_call = b.nop(m0)
            frame = []
            for i in range(nl1):
                if i < np1 and args[i] >= 0:
                    frame.append(b.copy(m0, cee(i), cal(args[i])))
                else:
                    frame.append(b.prim(m0, cee(i)))
            n_e, n_x = b.nop(m0), b.nop(m0)
            ret_copy = [b.copy(m0, lhs, cee(nl1 - 1))] if lhs is not None else []
            n_r = b.nop(m0)
            b.chain(b.entry(m0), *a_nodes, n_call, *frame, n_e, *c_nodes, n_x, *ret_copy,
                    n_r, *b_nodes, b.exit(m0))
            corr.update(CALL=n_call, RETSITE=n_r, E1=n_e, X1=n_x, E0=b.entry(m0), X0=b.exit(m0))
            cseq = [n_e, *c_nodes, n_x]
        else:
            c, r = b.call(m0, lhs, [cal(a) if a >= 0 else -1 for a in args], [m1])
            b.chain(b.entry(m0), *a_nodes, c)
            b.chain(r, *b_nodes, b.exit(m0))
            b.chain(b.entry(m1), *c_nodes, b.exit(m1))
            corr.update(CALL=c, RETSITE=r, E1=b.entry(m1), X1=b.exit(m1), E0=b.entry(m0),
                        X0=b.exit(m0))
            cseq = [b.entry(m1), *c_nodes, b.exit(m1)]
        # same extra branches inside C in both programs (between C statements / to exit)
        for (u, v) in c_branches:
            i = int(u * (len(cseq) - 2)) + 1      # a C statement (not entry/exit)
            j = int(v * (len(cseq) - 1)) + 1      # a later-or-earlier C statement or exit
            i = min(i, len(cseq) - 2)
            b.edge(cseq[i], cseq[min(j, len(cseq) - 1)])
        if loop:
            b.edge(b_nodes[-1], a_nodes[0])
        b.set_module(d, insts=list(range(1, len(b.inst_type))), statics=list(range(b.n_statics)))
        b.add_entry(m0)
        return b.build(name=f"inline_{'inl' if inline else 'call'}_{seed}"), corr

    P, cP = make(False)
    Q, cQ = make(True)
    pairs = {}
    for key, n in cP.items():
        side = "callee" if key[1:].isdigit() and key[0] == "C" or key in ("E1", "X1") else "caller"
        pairs[n] = (cQ[key], side)
    info = dict(nl0=nl0, nl1=nl1)
    return P, Q, pairs, info
