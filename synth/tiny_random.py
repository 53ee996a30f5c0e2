"""Seeded random *tiny* ICFGs (tens of nodes) for brute-force and property tests.

Input generator only (no method arithmetic).  Every node kind and edge kind of
SURVEY §8(c) C2/C3 appears: multi-target calls, recursion, loops, several
modules with partial instance/static pools (so CALL/RET projection drops
facts), statics, heap fields and arrays.
"""
from __future__ import annotations

import random
from typing import List

from .icfg import (ALOAD, ASTORE, COPY, CONST, F_ARR, FLOAD, FSTORE, NEW, NOP, PRIM,
                   RETV, SLOAD, SSTORE, E_INTRA, Icfg, IcfgBuilder)

_STMT_KINDS = [NOP, PRIM, CONST, NEW, COPY, SLOAD, SSTORE, RETV, FLOAD, FSTORE,
               ALOAD, ASTORE, "CALL"]


def random_tiny(seed: int, n_methods: int = None, n_modules: int = None,
                max_stmts: int = 5, full_pools: bool = False,
                kinds: List = None, allow_calls: bool = True, wide_pad: int = 0) -> Icfg:
    """wide_pad > 0 adds that many never-allocated instances to every module pool (half with
    lower gids than the real sites, half higher), so pools exceed 64 instances and the CUDA
    path takes its wide-block (row-occupancy) route with sites straddling word boundaries."""
    rng = random.Random(seed)
    n_fields = rng.randint(1, 3)                 # field 0 = F_ARR
    b = IcfgBuilder(n_fields=n_fields)
    n_types = rng.randint(1, 3)
    types = [b.add_type(rng.sample(range(n_fields), rng.randint(1, n_fields)))
             for _ in range(n_types)]
    n_statics = rng.randint(0, 2)
    for _ in range(n_statics):
        b.add_static()
    pad_lo = [b.add_instance(rng.choice(types)) for _ in range(wide_pad // 2)]
    M = n_methods or rng.randint(1, 3)
    D = n_modules or rng.randint(1, min(2, M))
    mods = [b.add_module() for _ in range(D)]
    meths = []
    for m in range(M):
        d = mods[m % D] if m < D else rng.choice(mods)
        np_ = rng.choice((0, 0, 1, 1, 2, 2, 3, 4, 5))       # arity 0..5
        nl = np_ + rng.randint(1, 2) + 1
        meths.append(b.add_method(d, np_, nl))
    kinds = kinds or _STMT_KINDS
    if not allow_calls:
        kinds = [k for k in kinds if k != "CALL"]
    mod_sites = {d: [] for d in mods}
    mod_stat_used = {d: set() for d in mods}
    for m in meths:
        d = b.methods[m].module
        nl = b.methods[m].n_locals
        loc = lambda: b.L(m, rng.randrange(nl - 1)) if nl > 1 else b.L(m, 0)  # non-RET locals
        seq = [b.entry(m)]
        heads = []            # (first, last) node of each statement for extra edges
        for _ in range(rng.randint(1, max_stmts)):
            k = rng.choice(kinds)
            if k == "CALL":
                np_ = rng.choice(sorted({b.methods[t].n_params for t in meths}))
                cands = [t for t in meths if b.methods[t].n_params == np_]
                targets = rng.sample(cands, rng.randint(1, min(2, len(cands))))
                lhs = loc() if rng.random() < 0.7 else None
                if np_ >= 2 and rng.random() < 0.35:     # one local passed as several actuals
                    rep = loc()
                    args = [rep if rng.random() < 0.8 else (-1 if rng.random() < 0.5 else loc())
                            for _ in range(np_)]
                else:
                    args = [loc() if rng.random() < 0.8 else -1 for _ in range(np_)]
                c, r = b.call(m, lhs, args, targets)
                heads.append((c, r))
                seq.append((c, r))
                continue
            if k in (SLOAD, SSTORE) and n_statics == 0:
                k = COPY
            if k == NOP:
                n = b.nop(m)
            elif k == PRIM:
                n = b.prim(m, loc())
            elif k == CONST:
                if rng.random() < 0.3:
                    n = b.const(m, loc(), 0)
                else:
                    o = b.add_instance(rng.choice(types))
                    mod_sites[d].append(o)
                    n = b.const(m, loc(), o)
            elif k == NEW:
                o = b.add_instance(rng.choice(types))
                mod_sites[d].append(o)
                n = b.new(m, loc(), o)
            elif k == COPY:
                n = b.copy(m, loc(), loc())
            elif k == SLOAD:
                g = rng.randrange(n_statics); mod_stat_used[d].add(g)
                n = b.sload(m, loc(), b.S(g))
            elif k == SSTORE:
                g = rng.randrange(n_statics); mod_stat_used[d].add(g)
                n = b.sstore(m, b.S(g), loc())
            elif k == RETV:
                n = b.retv(m, loc())
            elif k == FLOAD:
                n = b.fload(m, loc(), loc(), rng.randrange(n_fields))
            elif k == FSTORE:
                n = b.fstore(m, loc(), rng.randrange(n_fields), loc())
            elif k == ALOAD:
                n = b.aload(m, loc(), loc())
            elif k == ASTORE:
                n = b.astore(m, loc(), loc())
            else:
                raise AssertionError(k)
            heads.append((n, n))
            seq.append((n, n))
        seq.append(b.exit(m))
        # fall-through chain
        prev_last = seq[0]
        for item in seq[1:]:
            first, last = (item, item) if isinstance(item, int) else item
            b.edge(prev_last, first, E_INTRA)
            prev_last = last
        # extra branches / back edges (from a statement's last node, never from CALL)
        for _ in range(rng.randint(0, 2)):
            if not heads:
                break
            src = rng.choice(heads)[1]
            dst = rng.choice(heads + [(b.exit(m), b.exit(m))])[0]
            b.edge(src, dst, E_INTRA)
    pad_hi = [b.add_instance(rng.choice(types)) for _ in range(wide_pad - wide_pad // 2)]
    all_insts = list(range(1, len(b.inst_type)))
    for d in mods:
        extra = [] if full_pools else [o for o in all_insts if rng.random() < 0.5]
        insts = all_insts if full_pools else mod_sites[d] + extra
        stats = list(range(n_statics)) if (full_pools or rng.random() < 0.5) else \
            sorted(mod_stat_used[d] | {g for g in range(n_statics) if rng.random() < 0.5})
        b.set_module(d, insts=list(insts) + pad_lo + pad_hi, statics=stats)
    b.add_entry(meths[0])
    if M > 1 and rng.random() < 0.3:
        b.add_entry(meths[-1])
    return b.build(name=f"tiny_random_{seed}")
