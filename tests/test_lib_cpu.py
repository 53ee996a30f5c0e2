"""CPU-side checks of the C-ABI library (no GPU needed): it loads, exports every symbol that
include/gdroid.h declares, and its loader rejects invalid inputs with the documented status
before touching the device."""
from __future__ import annotations

import copy
import ctypes as C
import os
import re

import numpy as np
import pytest

import paper_conf_ipps_yuwobby20_b200 as gd
from paper_conf_ipps_yuwobby20_b200._binding import GdroidError
from programs import tiny, tiny2

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def declared_functions():
    src = open(os.path.join(ROOT, "include", "gdroid.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(gdroid_[a-z_]+)\s*\(", src)))


def test_header_symbols_exported():
    L = gd.lib()
    names = declared_functions()
    assert len(names) >= 12
    for nm in names:
        assert hasattr(L, nm), nm
    assert L.gdroid_abi_version() == 2


def _load_status(g):
    try:
        gd.load(g)
    except GdroidError as e:
        return e.code
    return 0


def _mut(g, **kw):
    h = copy.deepcopy(g)
    for k, v in kw.items():
        setattr(h, k, v)
    return h


def test_loader_rejects_invalid():
    g = tiny()[0]
    # arity mismatch (V6)
    mp = g.method_n_params.copy(); mp[1] = 2
    ml = g.method_n_locals.copy(); ml[1] = 4
    assert _load_status(_mut(g, method_n_params=mp, method_n_locals=ml)) == -1
    # NEW site outside its module pool (V1)
    mi = g.module_insts[g.module_insts != 3].copy()
    assert _load_status(_mut(g, module_insts=mi, module_inst_ptr=np.array([0, len(mi)], np.uint64))) == -2
    # static not visible (V2)
    assert _load_status(_mut(g, module_statics=np.zeros(0, np.uint32),
                             module_static_ptr=np.array([0, 0], np.uint64))) == -2
    # operand local of another method (V4)
    ops = g.node_ops.copy(); ops[9, 1] = 6     # n5: z = x  ->  z = t (a local of m1)
    assert _load_status(_mut(g, node_ops=ops)) == -2
    # RET edge re-targeted to a non-RETSITE (V5)
    ek = g.edge_kind.copy(); col = g.col.copy()
    e = int(np.nonzero(ek == 2)[0][0]); col[e] = 7
    assert _load_status(_mut(g, col=col)) == -1
    # CSR not monotone
    rp = g.row_ptr.copy(); rp[3], rp[4] = rp[4], rp[3]
    if rp[3] > rp[4]:
        assert _load_status(_mut(g, row_ptr=rp)) == -1
    # pool without NULL
    g2 = tiny2()[0]
    mi2 = g2.module_insts.copy(); mi2[0] = 1
    assert _load_status(_mut(g2, module_insts=mi2)) in (-1, -2)


def test_loader_size_limits():
    """GDROID_E_LIMIT (include/gdroid.h): > 512 instances in one module pool, a wide block of
    > 1024 rows, an out-degree > 32768 — all rejected by host validation before the device."""
    from synth import IcfgBuilder

    def app(n_inst=1, n_stat=0, fanout=1):
        b = IcfgBuilder(n_fields=1)
        t = b.add_type([0])
        for _ in range(n_stat):
            b.add_static()
        insts = [b.add_instance(t) for _ in range(n_inst)]
        d = b.add_module()
        m = b.add_method(d, 0, 2)
        n = b.nop(m)
        for _ in range(fanout):
            b.edge(b.entry(m), n)
        b.edge(n, b.exit(m))
        b.set_module(d, insts=insts, statics=list(range(n_stat)))
        b.add_entry(m)
        return b.build()

    assert _load_status(app(n_inst=513)) == -8             # pool > 512 instances
    assert _load_status(app(n_inst=100, n_stat=1100)) == -8 # wide block (> 64 instances) of > 1024 rows
    assert _load_status(app(fanout=32769)) == -8            # out-degree > 32768
    assert _load_status(app(n_inst=100, n_stat=10, fanout=3)) not in (-1, -2, -8)   # within limits


def test_null_handles_rejected():
    """Every entry point taking a handle rejects NULL with GDROID_E_INVALID (no device needed)."""
    L = gd.lib()
    n = C.c_uint64(0)
    assert L.gdroid_debug_tables(None, 0, None, 0, C.byref(n)) == -1
    assert L.gdroid_release_facts(None) == -1
    assert L.gdroid_n_apps(None) == 0
    assert L.gdroid_fact_bytes(None) == 0
    L.gdroid_free(None)                                   # accepts NULL
