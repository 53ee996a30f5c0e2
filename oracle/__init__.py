"""ctypes wrapper of the CPU oracle (oracle/oracle.cpp).

TEST INFRASTRUCTURE ONLY: imported by tests/, ``__graft_entry__.smoke()`` and
bench.py's ``cpu_baseline`` / ``--impl reference`` legs.  The product package
``paper_conf_ipps_yuwobby20_b200`` never imports this module, and this module
never imports the product package.  Input arrays come from ``synth`` (the
shared, arithmetic-free input module).

Parity status per function:
  * worklist fixed point (``build``)       pinned: Kleene brute force, Fig. 2
    rounds, order independence, post-fixpoint, golden tiny
  * node transfer functions (C2)         pinned: textbook reductions
    (reaching definitions, Andersen points-to) + hand-computed tiny golden
  * edge transforms CALL/RET/C2R (C3)    pinned: inlining law + golden tiny +
    projection containment / full-pool identity
  * ``digests`` (C8)                     pinned: recomputed from pairs in
    tests/test_oracle_pins.py with an independent Python splitmix64
  * ``mer_merge`` (Fig. 7)               pinned: Fig. 7 example
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess
import threading
from typing import List, Optional, Tuple

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.cpp")
_HDR = os.path.join(_HERE, "oracle.h")
_LIB = os.path.join(_HERE, "liboracle.so")
_lock = threading.Lock()
_lib = None


def build(force: bool = False) -> str:
    """Compile liboracle.so (plain g++ -O2, single-threaded code)."""
    with _lock:
        newest = max(os.path.getmtime(_SRC), os.path.getmtime(_HDR))
        if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < newest:
            tmp = _LIB + f".tmp{os.getpid()}"
            subprocess.check_call(["g++", "-O2", "-std=c++17", "-shared", "-fPIC",
                                   "-o", tmp, _SRC])
            os.replace(tmp, _LIB)
    return _LIB


class _Icfg(C.Structure):
    _fields_ = [(n, C.c_uint32) for n in ("n_nodes", "n_methods", "n_modules", "n_types",
                                           "n_instances", "n_statics", "n_fields", "n_entries")] + [
        ("n_edges", C.c_uint64),
        ("row_ptr", C.c_void_p), ("col", C.c_void_p), ("edge_kind", C.c_void_p),
        ("node_kind", C.c_void_p), ("node_method", C.c_void_p), ("node_ops", C.c_void_p),
        ("call_arg_ptr", C.c_void_p), ("call_args", C.c_void_p),
        ("method_entry", C.c_void_p), ("method_exit", C.c_void_p), ("method_module", C.c_void_p),
        ("method_n_locals", C.c_void_p), ("method_n_params", C.c_void_p),
        ("module_inst_ptr", C.c_void_p), ("module_insts", C.c_void_p),
        ("module_static_ptr", C.c_void_p), ("module_statics", C.c_void_p),
        ("inst_type", C.c_void_p),
        ("type_field_ptr", C.c_void_p), ("type_fields", C.c_void_p),
        ("entries", C.c_void_p),
    ]


def lib():
    global _lib
    if _lib is None:
        build()
        L = C.CDLL(_LIB)
        P = C.c_void_p
        L.oracle_build.argtypes = [P, C.c_int, C.c_uint64, C.POINTER(P)]
        L.oracle_build.restype = C.c_int
        L.oracle_free.argtypes = [P]
        L.oracle_last_error.restype = C.c_char_p
        L.oracle_visits.argtypes = [P]; L.oracle_visits.restype = C.c_uint64
        L.oracle_seconds.argtypes = [P]; L.oracle_seconds.restype = C.c_double
        L.oracle_total_pairs.argtypes = [P]; L.oracle_total_pairs.restype = C.c_uint64
        L.oracle_all_pairs.argtypes = [P, P, P]
        L.oracle_digests.argtypes = [P, P, P]
        L.oracle_check_postfix.argtypes = [P, P]; L.oracle_check_postfix.restype = C.c_uint64
        L.oracle_bsp_rounds.argtypes = [P, P, C.c_uint64, P, C.c_uint64]
        L.oracle_bsp_rounds.restype = C.c_int64
        L.oracle_mer_merge.argtypes = [P, C.c_uint64, P, C.c_uint64, P, C.c_uint64, P]
        L.oracle_mer_merge.restype = C.c_uint64
        _lib = L
    return _lib


def _ptr(a: np.ndarray):
    return a.ctypes.data_as(C.c_void_p) if a.size else None


def _desc(g) -> Tuple[_Icfg, list]:
    keep = []
    d = _Icfg()
    d.n_nodes, d.n_methods, d.n_modules = g.n_nodes, g.n_methods, g.n_modules
    d.n_types, d.n_instances, d.n_statics = g.n_types, g.n_instances, g.n_statics
    d.n_fields, d.n_entries, d.n_edges = g.n_fields, g.n_entries, g.n_edges
    for nm in ("row_ptr", "col", "edge_kind", "node_kind", "node_method", "node_ops",
               "call_arg_ptr", "call_args", "method_entry", "method_exit", "method_module",
               "method_n_locals", "method_n_params", "module_inst_ptr", "module_insts",
               "module_static_ptr", "module_statics", "inst_type", "type_field_ptr",
               "type_fields", "entries"):
        a = np.ascontiguousarray(getattr(g, nm))
        keep.append(a)
        setattr(d, nm, _ptr(a))
    return d, keep


class OracleError(RuntimeError):
    def __init__(self, code, msg):
        super().__init__(f"oracle status {code}: {msg}")
        self.code = code


class OracleResult:
    """IN(n) for every node, as sorted packed pairs (slot_gid << 32 | inst_gid)."""

    def __init__(self, handle, n_nodes):
        self._h = handle
        self.n_nodes = n_nodes
        L = lib()
        self.visits = int(L.oracle_visits(handle))
        self.seconds = float(L.oracle_seconds(handle))
        tot = int(L.oracle_total_pairs(handle))
        self.ptr = np.zeros(n_nodes + 1, dtype=np.uint64)
        self.pairs = np.zeros(max(tot, 1), dtype=np.uint64)[:tot]
        L.oracle_all_pairs(handle, _ptr(self.ptr), _ptr(self.pairs) if tot else None)
        self.node_digest = np.zeros(n_nodes, dtype=np.uint64)
        app = C.c_uint64(0)
        L.oracle_digests(handle, _ptr(self.node_digest), C.byref(app))
        self.app_digest = int(app.value)

    def facts(self, n: int) -> np.ndarray:
        return self.pairs[int(self.ptr[n]):int(self.ptr[n + 1])]

    def fact_set(self, n: int) -> set:
        return {(int(p) >> 32, int(p) & 0xFFFFFFFF) for p in self.facts(n)}

    def __del__(self):
        if getattr(self, "_h", None) is not None and _lib is not None:
            _lib.oracle_free(self._h)
            self._h = None


def build_idfg(g, order: int = 0, seed: int = 0) -> OracleResult:
    """Least fixed point by Alg. 1's worklist (order 0 FIFO / 1 LIFO / 2 random)."""
    L = lib()
    d, keep = _desc(g)
    h = C.c_void_p()
    rc = L.oracle_build(C.byref(d), order, seed, C.byref(h))
    if rc != 0:
        raise OracleError(rc, L.oracle_last_error().decode())
    r = OracleResult(h, g.n_nodes)
    r._g_keep = (d, keep)
    return r


def run_timed(g, order: int = 0):
    """The oracle's fixed point with only (seconds, visits, app digest) returned — no pair
    copy-out; used by bench.py's cpu_baseline / --impl reference legs (thread pools: the
    ctypes call releases the GIL and the oracle keeps no shared mutable state)."""
    L = lib()
    d, keep = _desc(g)
    h = C.c_void_p()
    rc = L.oracle_build(C.byref(d), order, 0, C.byref(h))
    if rc != 0:
        raise OracleError(rc, L.oracle_last_error().decode())
    try:
        app = C.c_uint64(0)
        L.oracle_digests(h, None, C.byref(app))
        return float(L.oracle_seconds(h)), int(L.oracle_visits(h)), int(app.value)
    finally:
        L.oracle_free(h)


def check_postfix(g, r: OracleResult) -> int:
    d, keep = _desc(g)
    return int(lib().oracle_check_postfix(C.byref(d), r._h))


def bsp_rounds(g, max_total: int = 1 << 20) -> List[List[int]]:
    L = lib()
    d, keep = _desc(g)
    seq = np.zeros(max_total, dtype=np.uint32)
    lens = np.zeros(max_total, dtype=np.uint32)
    nr = L.oracle_bsp_rounds(C.byref(d), _ptr(seq), max_total, _ptr(lens), max_total)
    if nr < 0:
        raise OracleError(nr, L.oracle_last_error().decode())
    out, k = [], 0
    for i in range(nr):
        out.append(seq[k:k + lens[i]].tolist())
        k += int(lens[i])
    return out


def mer_merge(worklist, dests) -> Tuple[int, List[int]]:
    L = lib()
    wl = np.asarray(worklist, dtype=np.uint32)
    ds = np.asarray(dests, dtype=np.uint32)
    cap = len(wl) + len(ds)
    nxt = np.zeros(max(cap, 1), dtype=np.uint32)
    head = C.c_uint64(0)
    n = L.oracle_mer_merge(_ptr(wl), len(wl), _ptr(ds), len(ds), _ptr(nxt), cap, C.byref(head))
    return int(head.value), nxt[:n].tolist()
