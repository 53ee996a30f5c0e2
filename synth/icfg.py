"""ICFG input container and a builder for hand-written programs.

This module is INPUT plumbing shared by the oracle (``oracle/``) and the CUDA
path (``paper_conf_ipps_yuwobby20_b200``).  It holds the array layout of an
ICFG (the paper's ``h_icfg`` + ``h_stmt`` + the pre-determined slot/instance
pools, Alg. 2 l.1-2, §IV-A) and nothing of
the method's arithmetic: no transfer function, no union, no fixed point.

Array layout (mirrors ``gdroid_icfg_desc`` in include/gdroid.h):

* nodes: ``node_kind`` u8[N], ``node_method`` u32[N], ``node_ops`` i32[N,4]
  = {op0 (lhs slot gid), op1 (rhs slot gid), op2 (field id), op3 (instance gid
  or, for RETSITE, its CALL node id)}; -1 = none.
* CSR successors: ``row_ptr`` u64[N+1], ``col`` u32[E], ``edge_kind`` u8[E].
* call arguments: ``call_arg_ptr`` u64[N+1], ``call_args`` i32[...] (local slot
  gid of the actual, or -1 for a non-reference actual), non-empty only for CALL.
* methods: entry/exit node, module, n_locals (params first, RET last), n_params.
* modules: instance pool ``module_insts`` (sorted gids, must contain 0 = NULL)
  and visible statics ``module_statics`` (sorted static indices), CSR.
* instances: ``inst_type`` i32[I] (-1 for NULL = gid 0).
* types: ``type_fields`` (sorted field ids) CSR.  Field id 0 is ``F_ARR``.
* ``entries``: ENTRY nodes of the component environment methods (Eq. 1,
  PAPER.md:351-355; one per component).

Slot gids (SURVEY §8(b) conventions): locals method-major
``local_base[m] + i``; statics ``L_total + g``; heap slots
``L_total + G + heap_base[o] + ordinal(f in F(t(o)))``.
"""
from __future__ import annotations

import json
from dataclasses import dataclass, field
from typing import Dict, List, Optional, Sequence, Tuple

import numpy as np

# ---- node kinds (paper statement/expression kinds PAPER.md:703-716)
NOP, ENTRY, EXIT, RETSITE, CALL, PRIM, CONST, NEW, COPY, SLOAD, SSTORE, RETV, \
    FLOAD, FSTORE, ALOAD, ASTORE = range(16)
KIND_NAMES = ["NOP", "ENTRY", "EXIT", "RETSITE", "CALL", "PRIM", "CONST", "NEW",
              "COPY", "SLOAD", "SSTORE", "RETV", "FLOAD", "FSTORE", "ALOAD",
              "ASTORE"]
# ---- edge kinds
E_INTRA, E_CALL, E_RET, E_C2R = range(4)
EDGE_NAMES = ["INTRA", "CALL", "RET", "C2R"]
# ---- the array pseudo-field
F_ARR = 0

ARRAY_FIELDS = [
    ("row_ptr", np.uint64), ("col", np.uint32), ("edge_kind", np.uint8),
    ("node_kind", np.uint8), ("node_method", np.uint32), ("node_ops", np.int32),
    ("call_arg_ptr", np.uint64), ("call_args", np.int32),
    ("method_entry", np.uint32), ("method_exit", np.uint32),
    ("method_module", np.uint32), ("method_n_locals", np.uint32),
    ("method_n_params", np.uint32),
    ("module_inst_ptr", np.uint64), ("module_insts", np.uint32),
    ("module_static_ptr", np.uint64), ("module_statics", np.uint32),
    ("inst_type", np.int32),
    ("type_field_ptr", np.uint64), ("type_fields", np.uint32),
    ("entries", np.uint32),
]


@dataclass
class Icfg:
    """Plain arrays of one app's ICFG (see module docstring)."""
    n_statics: int
    n_fields: int
    row_ptr: np.ndarray
    col: np.ndarray
    edge_kind: np.ndarray
    node_kind: np.ndarray
    node_method: np.ndarray
    node_ops: np.ndarray
    call_arg_ptr: np.ndarray
    call_args: np.ndarray
    method_entry: np.ndarray
    method_exit: np.ndarray
    method_module: np.ndarray
    method_n_locals: np.ndarray
    method_n_params: np.ndarray
    module_inst_ptr: np.ndarray
    module_insts: np.ndarray
    module_static_ptr: np.ndarray
    module_statics: np.ndarray
    inst_type: np.ndarray
    type_field_ptr: np.ndarray
    type_fields: np.ndarray
    entries: np.ndarray
    name: str = "app"

    def __post_init__(self):
        for nm, dt in ARRAY_FIELDS:
            a = np.ascontiguousarray(np.asarray(getattr(self, nm), dtype=dt))
            if nm == "node_ops":
                a = a.reshape(-1, 4)
            setattr(self, nm, a)

    # sizes -----------------------------------------------------------------
    @property
    def n_nodes(self) -> int: return int(self.node_kind.shape[0])
    @property
    def n_edges(self) -> int: return int(self.col.shape[0])
    @property
    def n_methods(self) -> int: return int(self.method_entry.shape[0])
    @property
    def n_modules(self) -> int: return int(self.module_inst_ptr.shape[0] - 1)
    @property
    def n_types(self) -> int: return int(self.type_field_ptr.shape[0] - 1)
    @property
    def n_instances(self) -> int: return int(self.inst_type.shape[0])
    @property
    def n_entries(self) -> int: return int(self.entries.shape[0])

    def nbytes(self) -> int:
        return sum(getattr(self, nm).nbytes for nm, _ in ARRAY_FIELDS)

    # numbering helpers (pure bookkeeping of the input format) -------------
    def local_base(self) -> np.ndarray:
        lb = np.zeros(self.n_methods + 1, dtype=np.int64)
        np.cumsum(self.method_n_locals, out=lb[1:])
        return lb

    def L_total(self) -> int:
        return int(self.method_n_locals.sum())

    # (de)serialisation for text fixtures ------------------------------------
    def to_json(self) -> str:
        d = {"name": self.name, "n_statics": self.n_statics, "n_fields": self.n_fields}
        for nm, _ in ARRAY_FIELDS:
            d[nm] = getattr(self, nm).reshape(-1).tolist()
        return json.dumps(d, separators=(",", ":"))

    @staticmethod
    def from_json(s: str) -> "Icfg":
        d = json.loads(s)
        kw = {nm: np.asarray(d[nm]) for nm, _ in ARRAY_FIELDS}
        return Icfg(n_statics=d["n_statics"], n_fields=d["n_fields"],
                    name=d.get("name", "app"), **kw)


# ---------------------------------------------------------------------------
# Builder for hand-written / small random programs.
# ---------------------------------------------------------------------------
class _Loc:
    __slots__ = ("m", "i")
    def __init__(self, m, i): self.m, self.i = m, i


class _Stat:
    __slots__ = ("g",)
    def __init__(self, g): self.g = g


@dataclass
class _Method:
    module: int
    n_params: int
    n_locals: int
    entry: int = -1
    exit: int = -1


class IcfgBuilder:
    """Incrementally build an :class:`Icfg`.

    Locals are referenced as ``b.L(m, i)`` and statics as ``b.S(g)``; they are
    resolved to slot gids by :meth:`build` (static gids depend on L_total).
    """

    def __init__(self, n_fields: int = 1):
        self.n_fields = n_fields
        self.types: List[List[int]] = []
        self.inst_type: List[int] = [-1]          # gid 0 = NULL
        self.n_statics = 0
        self.modules: List[Tuple[List[int], List[int]]] = []
        self.methods: List[_Method] = []
        self.kinds: List[int] = []
        self.nmeth: List[int] = []
        self.ops: List[list] = []
        self.args: Dict[int, list] = {}
        self.edges: List[Tuple[int, int, int]] = []
        self.entries: List[int] = []

    # universe ----------------------------------------------------------------
    def add_type(self, fields: Sequence[int]) -> int:
        for f in fields:
            assert 0 <= f < self.n_fields, "field id out of range"
        self.types.append(sorted(set(fields)))
        return len(self.types) - 1

    def add_instance(self, type_id: int) -> int:
        self.inst_type.append(type_id)
        return len(self.inst_type) - 1

    def add_static(self) -> int:
        self.n_statics += 1
        return self.n_statics - 1

    def add_module(self, insts: Sequence[int] = (), statics: Sequence[int] = ()) -> int:
        self.modules.append((sorted(set([0, *insts])), sorted(set(statics))))
        return len(self.modules) - 1

    def set_module(self, d: int, insts=None, statics=None):
        mi, ms = self.modules[d]
        if insts is not None:
            mi = sorted(set([0, *insts]))
        if statics is not None:
            ms = sorted(set(statics))
        self.modules[d] = (mi, ms)

    def add_method(self, module: int, n_params: int, n_locals: int) -> int:
        """n_locals counts params, temps and RET (last local)."""
        assert n_locals >= n_params + 1
        m = len(self.methods)
        self.methods.append(_Method(module, n_params, n_locals))
        self.methods[m].entry = self.node(m, ENTRY)
        self.methods[m].exit = self.node(m, EXIT)
        return m

    def L(self, m: int, i: int) -> _Loc:
        assert 0 <= i < self.methods[m].n_locals
        return _Loc(m, i)

    def RET(self, m: int) -> _Loc:
        return _Loc(m, self.methods[m].n_locals - 1)

    def S(self, g: int) -> _Stat:
        return _Stat(g)

    # nodes and edges ------------------------------------------------------------
    def node(self, m: int, kind: int, op0=None, op1=None, op2=None, op3=None) -> int:
        n = len(self.kinds)
        self.kinds.append(kind)
        self.nmeth.append(m)
        self.ops.append([op0, op1, op2, op3])
        return n

    def entry(self, m): return self.methods[m].entry
    def exit(self, m): return self.methods[m].exit

    def edge(self, a: int, b: int, kind: int = E_INTRA):
        self.edges.append((a, b, kind))

    def chain(self, *nodes: int):
        for a, b in zip(nodes[:-1], nodes[1:]):
            self.edge(a, b, E_INTRA)

    # statement shorthands -------------------------------------------------------
    def nop(self, m): return self.node(m, NOP)
    def prim(self, m, v): return self.node(m, PRIM, v)
    def const(self, m, v, inst): return self.node(m, CONST, v, None, None, inst)
    def new(self, m, v, inst): return self.node(m, NEW, v, None, None, inst)
    def copy(self, m, v, w): return self.node(m, COPY, v, w)
    def sload(self, m, v, g): return self.node(m, SLOAD, v, g)
    def sstore(self, m, g, w): return self.node(m, SSTORE, g, w)
    def retv(self, m, w): return self.node(m, RETV, None, w)
    def fload(self, m, v, w, f): return self.node(m, FLOAD, v, w, f)
    def fstore(self, m, v, f, w): return self.node(m, FSTORE, v, w, f)
    def aload(self, m, v, w): return self.node(m, ALOAD, v, w, F_ARR)
    def astore(self, m, v, w): return self.node(m, ASTORE, v, w, F_ARR)

    def call(self, m: int, lhs, args: Sequence, targets: Sequence[int]) -> Tuple[int, int]:
        """CALL node c + RETSITE r(c) with CALL/C2R/RET edges."""
        c = self.node(m, CALL, lhs)
        r = self.node(m, RETSITE, lhs, None, None, ("node", c))
        self.args[c] = list(args)
        for t in targets:
            assert self.methods[t].n_params == len(args), "arity mismatch"
            self.edge(c, self.methods[t].entry, E_CALL)
            self.edge(self.methods[t].exit, r, E_RET)
        self.edge(c, r, E_C2R)
        return c, r

    def add_entry(self, m: int):
        self.entries.append(self.methods[m].entry)

    # finalize -------------------------------------------------------------------
    def build(self, name: str = "app") -> Icfg:
        M = len(self.methods)
        lb = [0] * (M + 1)
        for m in range(M):
            lb[m + 1] = lb[m] + self.methods[m].n_locals
        L_total = lb[M]

        def res(x):
            if x is None:
                return -1
            if isinstance(x, _Loc):
                return lb[x.m] + x.i
            if isinstance(x, _Stat):
                return L_total + x.g
            if isinstance(x, tuple) and x[0] == "node":
                return x[1]
            return int(x)

        N = len(self.kinds)
        ops = np.array([[res(o) for o in op] for op in self.ops], dtype=np.int32).reshape(N, 4)
        # CSR, stable by source then insertion order
        order = sorted(range(len(self.edges)), key=lambda e: (self.edges[e][0], e))
        row_ptr = np.zeros(N + 1, dtype=np.uint64)
        for a, _, _ in self.edges:
            row_ptr[a + 1] += 1
        row_ptr = np.cumsum(row_ptr).astype(np.uint64)
        col = np.array([self.edges[e][1] for e in order], dtype=np.uint32)
        ek = np.array([self.edges[e][2] for e in order], dtype=np.uint8)
        cap = np.zeros(N + 1, dtype=np.uint64)
        cargs: List[int] = []
        for n in range(N):
            a = self.args.get(n, [])
            cargs.extend(res(x) for x in a)
            cap[n + 1] = cap[n] + len(a)
        mip = [0]; mis: List[int] = []; msp = [0]; mss: List[int] = []
        for insts, stats in self.modules:
            mis.extend(insts); mip.append(len(mis))
            mss.extend(stats); msp.append(len(mss))
        tfp = [0]; tfs: List[int] = []
        for fl in self.types:
            tfs.extend(fl); tfp.append(len(tfs))
        return Icfg(
            n_statics=self.n_statics, n_fields=self.n_fields, name=name,
            row_ptr=row_ptr, col=col, edge_kind=ek,
            node_kind=np.array(self.kinds, dtype=np.uint8),
            node_method=np.array(self.nmeth, dtype=np.uint32), node_ops=ops,
            call_arg_ptr=cap, call_args=np.array(cargs, dtype=np.int32),
            method_entry=[mm.entry for mm in self.methods],
            method_exit=[mm.exit for mm in self.methods],
            method_module=[mm.module for mm in self.methods],
            method_n_locals=[mm.n_locals for mm in self.methods],
            method_n_params=[mm.n_params for mm in self.methods],
            module_inst_ptr=mip, module_insts=mis,
            module_static_ptr=msp, module_statics=mss,
            inst_type=self.inst_type, type_field_ptr=tfp, type_fields=tfs,
            entries=self.entries)
