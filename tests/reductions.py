"""Independent textbook solvers used to pin the oracle (never shared with it).

* ``reaching_definitions`` — the classic iterative bit-vector solver
  (Aho, Lam, Sethi, Ullman, *Compilers* 2nd ed., §9.2.4): OUT[B] = gen_B ∪
  (IN[B] − kill_B), IN[B] = ∪ OUT[P] over reachable predecessors.
* ``andersen`` — flow-insensitive inclusion-based points-to (Andersen 1994),
  naive constraint iteration to the least solution.
Both speak symbolic slots ('L', m, i) / ('S', g) / ('H', o, f) (tests/kleene.Sym).
"""
from __future__ import annotations

from collections import defaultdict
from typing import Dict, Set

from synth.icfg import (ALOAD, ASTORE, CONST, COPY, F_ARR, FLOAD, FSTORE, NEW, PRIM, RETV,
                        SLOAD, SSTORE)

from kleene import Sym, reach


def reaching_definitions(g) -> Dict[int, Set]:
    """Returns {node: {(slot, inst)}} for reached nodes: the (var, inst) of every definition
    reaching the node's entry; PRIM definitions kill but carry no instance."""
    S = Sym(g)
    R = reach(g)
    defs = {}   # node -> (var, inst or None)
    for n in range(g.n_nodes):
        k = int(g.node_kind[n])
        if k in (NEW, CONST):
            defs[n] = (S.sym(int(g.node_ops[n][0])), int(g.node_ops[n][3]))
        elif k == PRIM:
            defs[n] = (S.sym(int(g.node_ops[n][0])), None)
    by_var = defaultdict(set)
    for n, (v, _) in defs.items():
        by_var[v].add(n)
    preds = defaultdict(list)
    for p in R:
        for e in range(int(g.row_ptr[p]), int(g.row_ptr[p + 1])):
            preds[int(g.col[e])].append(p)
    IN = {n: set() for n in R}
    OUT = {n: set() for n in R}
    changed = True
    while changed:
        changed = False
        for n in sorted(R):
            i = set().union(*(OUT[p] for p in preds[n])) if preds[n] else set()
            if n in defs:
                v = defs[n][0]
                o = (i - by_var[v]) | {n}
            else:
                o = set(i)
            if i != IN[n] or o != OUT[n]:
                IN[n], OUT[n] = i, o
                changed = True
    return {n: {(defs[d][0], defs[d][1]) for d in IN[n] if defs[d][1] is not None} for n in R}


def andersen(g) -> Set:
    """Least solution of Andersen's constraints for a single-method program; returns the
    set of (slot, inst) with inst ∈ pts(slot)."""
    S = Sym(g)
    pts = defaultdict(set)
    stmts = []
    for n in range(g.n_nodes):
        k = int(g.node_kind[n]); op = [int(x) for x in g.node_ops[n]]
        m = int(g.node_method[n])
        stmts.append((k, op, m))
    changed = True

    def add(slot, objs):
        nonlocal changed
        before = len(pts[slot])
        pts[slot] |= objs
        if len(pts[slot]) != before:
            changed = True

    while changed:
        changed = False
        for k, op, m in stmts:
            if k in (NEW, CONST):
                add(S.sym(op[0]), {op[3]})
            elif k in (COPY, SLOAD, SSTORE):
                add(S.sym(op[0]), set(pts[S.sym(op[1])]))
            elif k == RETV:
                add(S.ret(m), set(pts[S.sym(op[1])]))
            elif k in (FLOAD, ALOAD):
                f = F_ARR if k == ALOAD else op[2]
                for o1 in list(pts[S.sym(op[1])]):
                    h = S.heap(o1, f)
                    if h is not None:
                        add(S.sym(op[0]), set(pts[h]))
            elif k in (FSTORE, ASTORE):
                f = F_ARR if k == ASTORE else op[2]
                for o1 in list(pts[S.sym(op[0])]):
                    h = S.heap(o1, f)
                    if h is not None:
                        add(h, set(pts[S.sym(op[1])]))
    return {(s, o) for s, os in pts.items() for o in os}
