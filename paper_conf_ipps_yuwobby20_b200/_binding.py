"""ctypes binding of libgdroid.so — argument marshalling only.

Every step of the IDFG construction runs in the CUDA kernels behind the C ABI
(include/gdroid.h).  There is no CPU fallback: if the library is missing or no
CUDA device is usable, the calls raise.
"""
from __future__ import annotations

import ctypes as C
import os
from typing import List, Optional, Sequence, Tuple, Union

import numpy as np

from ._build import LIB

ABI_VERSION = 2
STATUS = {0: "OK", -1: "E_INVALID", -2: "E_POOL", -3: "E_OOM", -4: "E_CUDA", -5: "E_STATE",
          -6: "E_RANGE", -7: "E_SMALLBUF", -8: "E_LIMIT"}

_ARRAYS = ("row_ptr", "col", "edge_kind", "node_kind", "node_method", "node_ops", "call_arg_ptr",
           "call_args", "method_entry", "method_exit", "method_module", "method_n_locals",
           "method_n_params", "module_inst_ptr", "module_insts", "module_static_ptr",
           "module_statics", "inst_type", "type_field_ptr", "type_fields", "entries")


class IcfgDesc(C.Structure):
    _fields_ = [("abi_version", C.c_uint32)] + \
        [(n, C.c_uint32) for n in ("n_nodes", "n_methods", "n_modules", "n_types", "n_instances",
                                    "n_statics", "n_fields", "n_entries")] + \
        [("n_edges", C.c_uint64)] + [(n, C.c_void_p) for n in _ARRAYS]


class BuildOpts(C.Structure):
    _fields_ = [("async_", C.c_uint32), ("max_rounds", C.c_uint32), ("blocks", C.c_uint32),
                ("loop_mode", C.c_uint32), ("variant", C.c_uint32), ("no_byte_model", C.c_uint32),
                ("release_facts", C.c_uint32), ("keep_facts", C.c_uint32), ("reserve_sms", C.c_uint32)]


class BuildStats(C.Structure):
    _fields_ = [("rounds", C.c_uint64), ("node_visits", C.c_uint64), ("alg_bytes", C.c_uint64),
                ("dense_bytes", C.c_uint64), ("atomics", C.c_uint64), ("hist", C.c_uint64 * 3),
                ("build_ns", C.c_uint64), ("fixpoint_ns", C.c_uint64), ("h2d_ns", C.c_uint64),
                ("fact_bytes", C.c_uint64), ("kernel_launches", C.c_uint64)]

    def as_dict(self) -> dict:
        d = {k: int(getattr(self, k)) for k, _ in self._fields_ if k != "hist"}
        d["hist"] = [int(x) for x in self.hist]
        return d


VARIANTS = {"default": 0, "mat": 1, "mat_grp": 2, "gdroid": 3, "plain": 4, "cell": 5, "sbda": 6}   # gdroid_variant


def variant_id(v) -> int:
    return VARIANTS[v] if isinstance(v, str) else int(v)


class GdroidError(RuntimeError):
    def __init__(self, code: int, msg: str):
        super().__init__(f"gdroid {STATUS.get(code, code)}: {msg}")
        self.code = code


_lib = None


def lib():
    """Load the in-tree libgdroid.so (raises if it was not built)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB):
            raise RuntimeError(f"{LIB} is missing: run `python -c 'import __graft_entry__ as g; g.build()'`")
        L = C.CDLL(LIB)
        P = C.c_void_p
        L.gdroid_load_batch.argtypes = [P, C.c_uint32, C.c_int, P, C.POINTER(P)]
        L.gdroid_load_icfg.argtypes = [P, C.c_int, P, C.POINTER(P)]
        if hasattr(L, "gdroid_load_icfg_plain"):          # (absent in older builds used for A/B)
            L.gdroid_load_icfg_plain.argtypes = [P, C.c_int, P, C.POINTER(P)]
            L.gdroid_load_icfg_plain.restype = C.c_int
        L.gdroid_build_idfg.argtypes = [P, P, P]
        L.gdroid_sync.argtypes = [P, P]
        L.gdroid_release_facts.argtypes = [P]
        L.gdroid_stage_seeds.argtypes = [P, C.c_uint32, C.c_uint32, P, P, P]
        L.gdroid_read_reached.argtypes = [P, C.c_uint32, C.c_uint32, P, P]
        L.gdroid_read_nodes_facts.argtypes = [P, C.c_uint32, C.c_uint32, P, P, P, C.c_uint64]
        L.gdroid_export_facts.argtypes = [P, P, C.c_uint64]
        L.gdroid_import_facts.argtypes = [P, P, C.c_uint64]
        L.gdroid_stream_sync.argtypes = [P]
        L.gdroid_fact_bytes.argtypes = [P]
        L.gdroid_fact_bytes.restype = C.c_uint64
        L.gdroid_read_facts.argtypes = [P, C.c_uint32, P, C.c_uint64, P]
        L.gdroid_read_facts_in.argtypes = [P, C.c_uint32, C.c_uint32, P, C.c_uint64, P]
        L.gdroid_read_all_facts.argtypes = [P, C.c_uint32, P, P, C.c_uint64]
        L.gdroid_read_batch_facts.argtypes = [P, P, P, C.c_uint64]
        L.gdroid_read_batch_facts_async.argtypes = [P, P, P, C.c_uint64, P, C.c_uint32]
        L.gdroid_node_digests.argtypes = [P, P, P]
        L.gdroid_node_digests_in.argtypes = [P, C.c_uint32, P, P]
        L.gdroid_app_digests.argtypes = [P, P]
        L.gdroid_n_apps.argtypes = [P]
        L.gdroid_n_apps.restype = C.c_uint32
        L.gdroid_debug_trace.argtypes = [P, C.c_uint32]
        L.gdroid_debug_read_trace.argtypes = [P, P, C.c_uint64, P]
        L.gdroid_debug_trace.restype = C.c_int
        L.gdroid_debug_read_trace.restype = C.c_int
        L.gdroid_debug_phases.argtypes = [P, P]
        L.gdroid_debug_phases.restype = C.c_int
        L.gdroid_debug_tables.argtypes = [P, C.c_uint32, P, C.c_uint64, P]
        L.gdroid_debug_tables.restype = C.c_int
        L.gdroid_free.argtypes = [P]
        L.gdroid_free.restype = None
        L.gdroid_last_error.restype = C.c_char_p
        L.gdroid_abi_version.restype = C.c_uint32
        for f in ("gdroid_load_batch", "gdroid_load_icfg", "gdroid_build_idfg", "gdroid_sync", "gdroid_release_facts",
                  "gdroid_stage_seeds", "gdroid_read_reached", "gdroid_read_nodes_facts", "gdroid_export_facts", "gdroid_import_facts",
                  "gdroid_stream_sync",
                  "gdroid_read_facts", "gdroid_read_facts_in", "gdroid_read_all_facts", "gdroid_read_batch_facts",
                  "gdroid_read_batch_facts_async",
                  "gdroid_node_digests", "gdroid_node_digests_in", "gdroid_app_digests"):
            getattr(L, f).restype = C.c_int
        _lib = L
    return _lib


def _check(rc: int):
    if rc != 0:
        raise GdroidError(rc, lib().gdroid_last_error().decode())


def _ptr(a: np.ndarray):
    return a.ctypes.data_as(C.c_void_p) if a.size else None


def make_desc(g) -> Tuple[IcfgDesc, list]:
    """Marshal an Icfg-like object (synth.Icfg) into a gdroid_icfg_desc; returns (desc, keepalive)."""
    d = IcfgDesc()
    d.abi_version = ABI_VERSION
    d.n_nodes, d.n_methods, d.n_modules = g.n_nodes, g.n_methods, g.n_modules
    d.n_types, d.n_instances, d.n_statics = g.n_types, g.n_instances, g.n_statics
    d.n_fields, d.n_entries, d.n_edges = g.n_fields, g.n_entries, g.n_edges
    keep = []
    for nm in _ARRAYS:
        a = np.ascontiguousarray(getattr(g, nm))
        keep.append(a)
        setattr(d, nm, _ptr(a))
    return d, keep


class App:
    """A loaded batch of one or more apps on one device (owns device memory)."""

    def __init__(self, icfgs: Union[object, Sequence[object]], device: int = 0, stream: int = 0,
                 plain: bool = False):
        if not isinstance(icfgs, (list, tuple)):
            icfgs = [icfgs]
        L = lib()
        n = len(icfgs)
        if plain and n != 1:
            raise ValueError("the PLAIN variant takes one app per handle")
        arr = (IcfgDesc * n)()
        keep = []
        for i, g in enumerate(icfgs):
            d, k = make_desc(g)
            arr[i] = d
            keep.append(k)
        self._h = C.c_void_p()
        if plain:
            _check(L.gdroid_load_icfg_plain(C.cast(arr, C.c_void_p), device, C.c_void_p(stream),
                                            C.byref(self._h)))
        else:
            _check(L.gdroid_load_batch(C.cast(arr, C.c_void_p), n, device, C.c_void_p(stream),
                                       C.byref(self._h)))
        self.n_apps = n
        self.n_nodes = [g.n_nodes for g in icfgs]
        self.stats: Optional[dict] = None

    def build(self, max_rounds: int = 0, blocks: int = 0, loop_mode: int = 0,
              asynchronous: bool = False, variant=0, byte_model: bool = True,
              release_facts: bool = False, keep_facts: bool = False, reserve_sms: int = 0) -> Optional[dict]:
        o = BuildOpts(1 if asynchronous else 0, max_rounds, blocks, loop_mode, variant_id(variant),
                      0 if byte_model else 1, 1 if release_facts else 0, 1 if keep_facts else 0, reserve_sms)
        s = BuildStats()
        _check(lib().gdroid_build_idfg(self._h, C.byref(o), C.byref(s)))
        if asynchronous:
            return None
        self.stats = s.as_dict()
        return self.stats

    # ---- incremental builds / out-of-core sub-graphs (gdroid_stage_seeds & co.)
    def stage_seeds(self, nodes, ptr, pairs, k: int = 0):
        nodes = np.ascontiguousarray(nodes, dtype=np.uint32)
        ptr = np.ascontiguousarray(ptr, dtype=np.uint64)
        pairs = np.ascontiguousarray(pairs, dtype=np.uint64)
        assert len(ptr) == len(nodes) + 1
        _check(lib().gdroid_stage_seeds(self._h, k, len(nodes), _ptr(nodes), _ptr(ptr), _ptr(pairs)))

    def read_reached(self, nodes, k: int = 0) -> np.ndarray:
        nodes = np.ascontiguousarray(nodes, dtype=np.uint32)
        out = np.zeros(max(len(nodes), 1), dtype=np.uint8)
        _check(lib().gdroid_read_reached(self._h, k, len(nodes), _ptr(nodes), _ptr(out)))
        return out[:len(nodes)].astype(bool)

    def read_nodes_facts(self, nodes, k: int = 0) -> Tuple[np.ndarray, np.ndarray]:
        nodes = np.ascontiguousarray(nodes, dtype=np.uint32)
        L = lib()
        ptr = np.zeros(len(nodes) + 1, dtype=np.uint64)
        _check(L.gdroid_read_nodes_facts(self._h, k, len(nodes), _ptr(nodes), _ptr(ptr), None, 0))
        tot = int(ptr[-1])
        pairs = np.zeros(max(tot, 1), dtype=np.uint64)
        _check(L.gdroid_read_nodes_facts(self._h, k, len(nodes), _ptr(nodes), _ptr(ptr), _ptr(pairs), tot))
        return ptr, pairs[:tot]

    @property
    def fact_bytes(self) -> int:
        return int(lib().gdroid_fact_bytes(self._h))

    def export_facts(self, host: np.ndarray):
        assert host.flags.c_contiguous and host.nbytes == self.fact_bytes
        _check(lib().gdroid_export_facts(self._h, _ptr(host), host.nbytes))

    def import_facts(self, host: np.ndarray):
        assert host.flags.c_contiguous and host.nbytes == self.fact_bytes
        _check(lib().gdroid_import_facts(self._h, _ptr(host), host.nbytes))

    def stream_sync(self):
        _check(lib().gdroid_stream_sync(self._h))

    def release_facts(self):
        """gdroid_release_facts: return the fact store to the device pool (digests stay)."""
        _check(lib().gdroid_release_facts(self._h))

    def sync(self) -> dict:
        s = BuildStats()
        _check(lib().gdroid_sync(self._h, C.byref(s)))
        self.stats = s.as_dict()
        return self.stats

    def read_facts(self, node: int, k: int = 0) -> np.ndarray:
        L = lib()
        cnt = C.c_uint64(0)
        _check(L.gdroid_read_facts_in(self._h, k, node, None, 0, C.byref(cnt)))
        out = np.zeros(max(cnt.value, 1), dtype=np.uint64)
        _check(L.gdroid_read_facts_in(self._h, k, node, _ptr(out), cnt.value, C.byref(cnt)))
        return out[:cnt.value]

    def read_all_facts(self, k: int = 0, ptr_out: Optional[np.ndarray] = None,
                       pairs_buf=None) -> Tuple[np.ndarray, np.ndarray]:
        """All facts of app k (CSR ptr[n_nodes+1], pairs).  ptr_out: a caller uint64 array of
        n_nodes+1; pairs_buf: an object with .get(n) -> uint64 array of n (e.g. a reusable
        pinned buffer), else fresh numpy arrays."""
        L = lib()
        ptr = ptr_out if ptr_out is not None else np.zeros(self.n_nodes[k] + 1, dtype=np.uint64)
        assert ptr.dtype == np.uint64 and ptr.size == self.n_nodes[k] + 1 and ptr.flags.c_contiguous
        _check(L.gdroid_read_all_facts(self._h, k, _ptr(ptr), None, 0))
        tot = int(ptr[-1])
        pairs = pairs_buf.get(tot) if pairs_buf is not None else np.zeros(max(tot, 1), dtype=np.uint64)[:tot]
        _check(L.gdroid_read_all_facts(self._h, k, _ptr(ptr), _ptr(pairs) if tot else None, tot))
        return ptr, pairs[:tot]

    def read_batch_facts(self, ptr_buf=None, pairs_buf=None) -> Tuple[np.ndarray, np.ndarray]:
        """gdroid_read_batch_facts: (ptr[N_batch+1], pairs) over all apps of the handle; the
        buffers (objects with .get(n) -> uint64 array, e.g. reusable pinned memory) are
        optional."""
        L = lib()
        n = sum(self.n_nodes)
        ptr = ptr_buf.get(n + 1) if ptr_buf is not None else np.zeros(n + 1, dtype=np.uint64)
        _check(L.gdroid_read_batch_facts(self._h, _ptr(ptr), None, 0))
        tot = int(ptr[-1])
        pairs = pairs_buf.get(tot) if pairs_buf is not None else np.zeros(max(tot, 1), dtype=np.uint64)[:tot]
        _check(L.gdroid_read_batch_facts(self._h, _ptr(ptr), _ptr(pairs) if tot else None, tot))
        return ptr, pairs[:tot]

    def read_batch_facts_async(self, ptr: np.ndarray, pairs: np.ndarray, total: np.ndarray, blocks: int = 0):
        """gdroid_read_batch_facts_async: enqueue the whole-batch readback into PINNED buffers
        (ptr of n+1, pairs of any capacity, total of 1); complete with stream_sync()."""
        n = sum(self.n_nodes)
        assert ptr.dtype == np.uint64 and ptr.size >= n + 1 and total.size >= 1
        rc = lib().gdroid_read_batch_facts_async(self._h, _ptr(ptr), _ptr(pairs), pairs.size, _ptr(total), blocks)
        if rc == -7:
            return False                                   # pairs buffer too small (nothing copied)
        _check(rc)
        return True

    def node_digests(self, k: int = 0) -> Tuple[np.ndarray, int]:
        per = np.zeros(self.n_nodes[k], dtype=np.uint64)
        app = C.c_uint64(0)
        _check(lib().gdroid_node_digests_in(self._h, k, _ptr(per), C.byref(app)))
        return per, int(app.value)

    def app_digests(self) -> np.ndarray:
        out = np.zeros(self.n_apps, dtype=np.uint64)
        _check(lib().gdroid_app_digests(self._h, _ptr(out)))
        return out

    def set_trace(self, cap: int):
        _check(lib().gdroid_debug_trace(self._h, cap))

    def read_trace(self) -> np.ndarray:
        """Per-round (start ns, items, nodes) of the last build (diagnostics)."""
        n = C.c_uint64(0)
        _check(lib().gdroid_debug_read_trace(self._h, None, 0, C.byref(n)))
        buf = np.zeros(2 * max(n.value, 1), dtype=np.uint64)
        _check(lib().gdroid_debug_read_trace(self._h, _ptr(buf), buf.size, C.byref(n)))
        t = buf.reshape(-1, 2)[:n.value]
        return np.stack([t[:, 0], t[:, 1] >> 32, t[:, 1] & 0xFFFFFFFF], axis=1)

    def phases(self) -> np.ndarray:
        out = np.zeros(8, dtype=np.uint64)
        _check(lib().gdroid_debug_phases(self._h, _ptr(out)))
        return out

    def table(self, which: int) -> np.ndarray:
        """Raw bytes of one device table (gdroid_debug_tables; diagnostics)."""
        n = C.c_uint64(0)
        _check(lib().gdroid_debug_tables(self._h, which, None, 0, C.byref(n)))
        buf = np.zeros(max(n.value, 1), dtype=np.uint8)
        _check(lib().gdroid_debug_tables(self._h, which, _ptr(buf), buf.size, C.byref(n)))
        return buf[:n.value]

    def free(self):
        if getattr(self, "_h", None) is not None and self._h.value:
            lib().gdroid_free(self._h)
            self._h = C.c_void_p()

    def __del__(self):
        try:
            self.free()
        except Exception:
            pass


def load(icfgs, device: int = 0, stream: int = 0, plain: bool = False) -> App:
    """gdroid_load_batch (or gdroid_load_icfg_plain with plain=True: one app, every variant)."""
    return App(icfgs, device=device, stream=stream, plain=plain)
