"""Python wrapper of the C++ synthetic-app generator (synth/gen.cpp) and the config presets.

Configs follow BASELINE.json ``configs`` and DESIGN.md §6:
  tiny    hand-written (tests/golden/programs.py::tiny)
  small   ~500 methods, ~20K nodes, K=3 components, |Q|=64      (seed 1)
  median  ~5K methods, ~300K nodes, K=48 components, |Q|=64     (seed 2)
  worst   ~30K methods, ~2M nodes, K=1, deep chains, |Q|=256    (seed 3)
  corpus  1000 apps, LogNormal(median 300K nodes, sigma 0.9) in [20K, 2M], seeds 1000+i
Input construction only: no transfer function, union or fixed point lives here.
"""
from __future__ import annotations

import ctypes as C
import math
import os
import random
import subprocess
import threading
from dataclasses import dataclass, field, replace
from typing import List

import numpy as np

from .icfg import ARRAY_FIELDS, Icfg

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "gen.cpp")
_LIB = os.path.join(_HERE, "libgdrgen.so")
_lock = threading.Lock()
_lib = None
GEN_VERSION = 2   # 2: arity 0..8 with repeated actuals (round 2)


def build(force: bool = False) -> str:
    with _lock:
        if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
            tmp = _LIB + f".tmp{os.getpid()}"
            subprocess.check_call(["g++", "-O2", "-std=c++17", "-shared", "-fPIC", "-o", tmp, _SRC])
            os.replace(tmp, _LIB)
    return _LIB


class _Params(C.Structure):
    _fields_ = [("seed", C.c_uint64)] + [(n, C.c_uint32) for n in (
        "n_methods", "stmts_per_method", "n_components", "methods_per_module", "q_cap", "n_types",
        "n_fields", "fields_per_type", "statics_per_module", "temps_per_method", "call_span")] + [
        ("p_recursion", C.c_double), ("mix", C.c_double * 13)]


# statement mix (paper silent): PRIM COPY CONST NEW FLOAD FSTORE ALOAD ASTORE
# SLOAD SSTORE CALL NOP, then the branch probability of the structured-CFG generator.
DEFAULT_MIX = (8, 16, 8, 8, 10, 8, 2, 2, 4, 3, 15, 12, 0.12)


@dataclass
class GenConfig:
    name: str
    seed: int
    n_methods: int
    stmts_per_method: int
    n_components: int
    methods_per_module: int = 8
    q_cap: int = 64
    n_types: int = 0            # 0: n_methods // 4
    n_fields: int = 24
    fields_per_type: int = 2
    statics_per_module: int = 2
    temps_per_method: int = 10
    call_span: int = 24
    p_recursion: float = 0.02
    mix: tuple = DEFAULT_MIX


PRESETS = {
    "small": GenConfig("small", 1, 500, 45, 3),
    "median": GenConfig("median", 2, 5000, 66, 48),
    "worst": GenConfig("worst", 3, 30000, 90, 1, methods_per_module=16, q_cap=256,
                       fields_per_type=2, call_span=12, p_recursion=0.03),
}


def _lib_():
    global _lib
    if _lib is None:
        build()
        L = C.CDLL(_LIB)
        L.gen_app.argtypes = [C.c_void_p]
        L.gen_app.restype = C.c_void_p
        L.gen_arrays.argtypes = [C.c_void_p, C.c_void_p, C.c_void_p, C.c_void_p]
        L.gen_free.argtypes = [C.c_void_p]
        _lib = L
    return _lib


def generate(cfg: GenConfig) -> Icfg:
    L = _lib_()
    p = _Params()
    p.seed = cfg.seed
    p.n_methods, p.stmts_per_method, p.n_components = cfg.n_methods, cfg.stmts_per_method, cfg.n_components
    p.methods_per_module, p.q_cap = cfg.methods_per_module, cfg.q_cap
    p.n_types = cfg.n_types or max(4, cfg.n_methods // 4)
    p.n_fields, p.fields_per_type = cfg.n_fields, cfg.fields_per_type
    p.statics_per_module, p.temps_per_method, p.call_span = cfg.statics_per_module, cfg.temps_per_method, cfg.call_span
    p.p_recursion = cfg.p_recursion
    for i, x in enumerate(cfg.mix):
        p.mix[i] = float(x)
    h = L.gen_app(C.byref(p))
    if not h:
        raise MemoryError("generator failed")
    try:
        ptrs = (C.c_void_p * 21)()
        lens = (C.c_uint64 * 21)()
        sc = (C.c_uint64 * 4)()
        L.gen_arrays(h, ptrs, lens, sc)
        kw = {}
        for i, (nm, dt) in enumerate(ARRAY_FIELDS):
            n = int(lens[i])
            item = np.dtype(dt).itemsize
            if n == 0:
                kw[nm] = np.zeros(0, dtype=dt)
            else:
                buf = (C.c_char * (n * item)).from_address(ptrs[i])
                kw[nm] = np.frombuffer(buf, dtype=dt).copy()
        g = Icfg(n_statics=int(sc[0]), n_fields=int(sc[1]), name=f"{cfg.name}_s{cfg.seed}", **kw)
    finally:
        L.gen_free(h)
    return g


def preset(name: str, seed: int = None) -> Icfg:
    cfg = PRESETS[name]
    if seed is not None:
        cfg = replace(cfg, seed=seed)
    return generate(cfg)


# ---------------------------------------------------------------------------- corpus
def corpus_config(i: int) -> GenConfig:
    """App i of the 1000-app corpus (seed 1000+i): N ~ LogNormal(median 300K, sigma 0.9) clipped
    to [20K, 2M] nodes; methods = N/51 (median shape: ~51 nodes per method; worst shape ~67);
    K = max(1, round(N/6217))
    (Table I); the top 1% (N >= 99th percentile) use the worst-case shape."""
    rng = random.Random(1000 + i)
    n = math.exp(math.log(300_000) + 0.9 * rng.gauss(0.0, 1.0))
    n = int(min(max(n, 20_000), 2_000_000))
    if n >= 2_000_000:                            # clipped tail (~1.7%): worst-case shape
        return replace(PRESETS["worst"], name=f"corpus{i}", seed=1000 + i, n_methods=max(8, n // 67))
    methods = max(8, n // 51)
    k = max(1, round(n / 6217))
    return replace(PRESETS["median"], name=f"corpus{i}", seed=1000 + i, n_methods=methods,
                   n_components=min(k, methods))


def corpus_app(i: int) -> Icfg:
    return generate(corpus_config(i))


def corpus_sizes(n_apps: int = 1000) -> List[int]:
    """Estimated node counts (for LPT sharding before generation)."""
    return [corpus_config(i).n_methods * (67 if corpus_config(i).q_cap > 64 else 51)
            for i in range(n_apps)]
