"""Brute-force Kleene (Jacobi) solver — an independent pin of the oracle's worklist.

Written separately from oracle/oracle.cpp, in a different representation:
slots are symbolic tuples ('L', m, i) / ('S', g) / ('H', o, f), sets are Python
frozensets, and every node is recomputed simultaneously from ⊥ until nothing
changes (IN(n) = ⋃ T_e(f_p(IN(p))) over reached p; Kildall /
Kam-Ullman: the Jacobi sequence from ⊥ reaches the least fixed point).
Only for tiny inputs.
"""
from __future__ import annotations

from collections import deque
from typing import Dict, FrozenSet, Set, Tuple

import numpy as np

from synth.icfg import (ALOAD, ASTORE, CALL, CONST, COPY, E_C2R, E_CALL, E_INTRA, E_RET,
                        ENTRY, EXIT, F_ARR, FLOAD, FSTORE, NEW, NOP, PRIM, RETSITE, RETV,
                        SLOAD, SSTORE)


class Sym:
    """Symbolic view of an Icfg's slot numbering (independent re-derivation)."""

    def __init__(self, g):
        self.g = g
        self.lb = [0]
        for m in range(g.n_methods):
            self.lb.append(self.lb[-1] + int(g.method_n_locals[m]))
        self.Lt = self.lb[-1]
        self.fields = []
        for t in range(g.n_types):
            a, b = int(g.type_field_ptr[t]), int(g.type_field_ptr[t + 1])
            self.fields.append([int(x) for x in g.type_fields[a:b]])
        # heap gid table: walk instances in gid order, each field of its type in order
        self.heap_gid: Dict[Tuple[int, int], int] = {}
        self.gid_heap: Dict[int, Tuple[int, int]] = {}
        nxt = self.Lt + g.n_statics
        for o in range(g.n_instances):
            t = int(g.inst_type[o])
            if t < 0:
                continue
            for f in self.fields[t]:
                self.heap_gid[(o, f)] = nxt
                self.gid_heap[nxt] = (o, f)
                nxt += 1
        self.mod_insts = []
        self.mod_stats = []
        for d in range(g.n_modules):
            a, b = int(g.module_inst_ptr[d]), int(g.module_inst_ptr[d + 1])
            self.mod_insts.append({int(x) for x in g.module_insts[a:b]})
            a, b = int(g.module_static_ptr[d]), int(g.module_static_ptr[d + 1])
            self.mod_stats.append({int(x) for x in g.module_statics[a:b]})

    def sym(self, s: int):
        if s < 0:
            return None
        if s < self.Lt:
            m = next(m for m in range(self.g.n_methods) if self.lb[m] <= s < self.lb[m + 1])
            return ("L", m, s - self.lb[m])
        if s < self.Lt + self.g.n_statics:
            return ("S", s - self.Lt)
        o, f = self.gid_heap[s]
        return ("H", o, f)

    def gid(self, slot) -> int:
        if slot[0] == "L":
            return self.lb[slot[1]] + slot[2]
        if slot[0] == "S":
            return self.Lt + slot[1]
        return self.heap_gid[(slot[1], slot[2])]

    def heap(self, o: int, f: int):
        t = int(self.g.inst_type[o])
        if o == 0 or t < 0 or f not in self.fields[t]:
            return None
        return ("H", o, f)

    def ret(self, m: int):
        return ("L", m, int(self.g.method_n_locals[m]) - 1)

    def in_pool(self, m: int, slot, o: int) -> bool:
        d = int(self.g.method_module[m])
        if o not in self.mod_insts[d]:
            return False
        if slot[0] == "L":
            return slot[1] == m
        if slot[0] == "S":
            return slot[1] in self.mod_stats[d]
        return slot[1] in self.mod_insts[d]


def _pts(X, slot):
    return {o for (s, o) in X if s == slot}


def node_fn(S: Sym, n: int, X: FrozenSet) -> FrozenSet:
    g = S.g
    k = int(g.node_kind[n])
    op = [int(x) for x in g.node_ops[n]]
    m = int(g.node_method[n])
    if k in (NOP, ENTRY, EXIT, RETSITE, CALL):
        return X
    if k == PRIM:
        v = S.sym(op[0]); return frozenset(p for p in X if p[0] != v)
    if k in (CONST, NEW):
        v = S.sym(op[0]); return frozenset({p for p in X if p[0] != v} | {(v, op[3])})
    if k in (COPY, SLOAD):
        v, w = S.sym(op[0]), S.sym(op[1])
        return frozenset({p for p in X if p[0] != v} | {(v, o) for o in _pts(X, w)})
    if k == SSTORE:
        gg, w = S.sym(op[0]), S.sym(op[1])
        return frozenset(set(X) | {(gg, o) for o in _pts(X, w)})
    if k == RETV:
        r, w = S.ret(m), S.sym(op[1])
        return frozenset({p for p in X if p[0] != r} | {(r, o) for o in _pts(X, w)})
    if k in (FLOAD, ALOAD):
        v, w = S.sym(op[0]), S.sym(op[1])
        f = F_ARR if k == ALOAD else op[2]
        gen = set()
        for o1 in _pts(X, w):
            h = S.heap(o1, f)
            if h is not None:
                gen |= {(v, o2) for o2 in _pts(X, h)}
        return frozenset({p for p in X if p[0] != v} | gen)
    if k in (FSTORE, ASTORE):
        v, w = S.sym(op[0]), S.sym(op[1])
        f = F_ARR if k == ASTORE else op[2]
        gen = set()
        for o1 in _pts(X, v):
            h = S.heap(o1, f)
            if h is not None:
                gen |= {(h, o2) for o2 in _pts(X, w)}
        return frozenset(set(X) | gen)
    raise AssertionError(k)


def edge_fn(S: Sym, p: int, s: int, kind: int, Y: FrozenSet) -> Set:
    g = S.g
    glob = {q for q in Y if q[0][0] != "L"}
    if kind == E_INTRA:
        return set(Y)
    if kind == E_C2R:
        m = int(g.node_method[p])
        lhs = S.sym(int(g.node_ops[p][0]))
        return {q for q in Y if q[0][0] == "L" and q[0][1] == m and q[0] != lhs} | glob
    if kind == E_CALL:
        callee = int(g.node_method[s])
        a0, a1 = int(g.call_arg_ptr[p]), int(g.call_arg_ptr[p + 1])
        Z = set(glob)
        for j, a in enumerate(int(x) for x in g.call_args[a0:a1]):
            if a >= 0:
                Z |= {(("L", callee, j), o) for o in _pts(Y, S.sym(a))}
        return {q for q in Z if S.in_pool(callee, q[0], q[1])}
    if kind == E_RET:
        callee = int(g.node_method[p])
        caller = int(g.node_method[s])
        lhs = S.sym(int(g.node_ops[s][0]))
        Z = set(glob)
        if lhs is not None:
            Z |= {(lhs, o) for o in _pts(Y, S.ret(callee))}
        return {q for q in Z if S.in_pool(caller, q[0], q[1])}
    raise AssertionError(kind)


def reach(g) -> Set[int]:
    seen = set(int(e) for e in g.entries)
    dq = deque(seen)
    while dq:
        n = dq.popleft()
        for e in range(int(g.row_ptr[n]), int(g.row_ptr[n + 1])):
            s = int(g.col[e])
            if s not in seen:
                seen.add(s); dq.append(s)
    return seen


def kleene(g, max_iter: int = 10000):
    """Jacobi iteration from ⊥ restricted to Reach; returns {node: frozenset of sym pairs}."""
    S = Sym(g)
    R = reach(g)
    IN = {n: frozenset() for n in range(g.n_nodes)}
    for _ in range(max_iter):
        new = {n: set() for n in range(g.n_nodes)}
        for p in R:
            Y = node_fn(S, p, IN[p])
            for e in range(int(g.row_ptr[p]), int(g.row_ptr[p + 1])):
                s = int(g.col[e])
                new[s] |= edge_fn(S, p, s, int(g.edge_kind[e]), Y)
        new = {n: frozenset(v) for n, v in new.items()}
        if new == IN:
            return S, IN
        IN = new
    raise RuntimeError("Kleene iteration did not converge")


def to_sym(S: Sym, pairs) -> FrozenSet:
    return frozenset((S.sym(int(p) >> 32), int(p) & 0xFFFFFFFF) for p in pairs)
