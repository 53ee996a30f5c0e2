"""Hand-written golden programs (text fixtures are the *.expected files beside this).

* ``tiny``  — BASELINE.json configs[0]: one class/module, 3 methods, 1 call
  site, ≤16 slots and instances, every node kind of SURVEY §8(c) C2 and every
  edge kind of C3, containing the Fig. 2 shape (entry, diamond, loop back to
  the head).  m2 has no caller (reading A5: its nodes stay
  ∅) unless ``m2_entry`` lists it as a second component entry (A11).
  Expected sets (tiny.expected, tiny_m2.expected) were computed BY HAND from
  the C2/C3 tables (derivation in tiny.expected's header), not by any code.
* ``tiny2`` — two modules with partial pools: the CALL and RET projections π
  drop an out-of-pool instance, an invisible static and a heap fact
  (reading A9).  Hand-computed in tiny2.expected.
* ``fig2``  — the ICFG shape of Fig. 2: entry→L1→
  {L2,L4}; L2→L3; L4→L5; {L3,L5}→L6→L7→{L1, exit}; L7 is ``x = new T``.
"""
from __future__ import annotations

import os
from typing import Dict, Tuple

from synth.icfg import E_INTRA, Icfg, IcfgBuilder

HERE = os.path.dirname(os.path.abspath(__file__))


def tiny(m2_entry: bool = False):
    b = IcfgBuilder(n_fields=2)               # field 0 = ARR, field 1 = f
    F = 1
    T_A = b.add_type([F]); T_ARR = b.add_type([0]); T_STR = b.add_type([]); T_CLS = b.add_type([])
    o1 = b.add_instance(T_A); o2 = b.add_instance(T_A); o3 = b.add_instance(T_ARR)
    o4 = b.add_instance(T_STR); o5 = b.add_instance(T_CLS)
    g0 = b.add_static()
    d = b.add_module(insts=[o1, o2, o3, o4, o5], statics=[g0])
    m0 = b.add_method(d, 0, 5)   # x y z a RET0
    m1 = b.add_method(d, 1, 3)   # p t RET1
    m2 = b.add_method(d, 0, 2)   # u RET2
    x, y, z, a = (b.L(m0, i) for i in range(4))
    p, t = b.L(m1, 0), b.L(m1, 1)
    u = b.L(m2, 0)
    G = b.S(g0)
    lab = {"e0": b.entry(m0), "x0": b.exit(m0), "e1": b.entry(m1), "x1": b.exit(m1),
           "e2": b.entry(m2), "x2": b.exit(m2)}
    # m0
    lab["n2"] = b.new(m0, x, o1)
    lab["n3"] = b.const(m0, y, o4)
    lab["n4"] = b.nop(m0)
    lab["n5"] = b.copy(m0, z, x)
    lab["n6"] = b.const(m0, z, 0)
    lab["n7"] = b.fstore(m0, x, F, y)
    lab["n8"] = b.sstore(m0, G, z)
    lab["n9"] = b.new(m0, a, o3)
    lab["n10"] = b.astore(m0, a, x)
    lab["n11"], lab["n12"] = b.call(m0, y, [x], [m1])
    lab["n13"] = b.aload(m0, z, a)
    lab["n14"] = b.sload(m0, y, G)
    lab["n15"] = b.prim(m0, a)
    lab["n16"] = b.nop(m0)
    lab["n17"] = b.retv(m0, z)
    L = lab
    b.chain(L["e0"], L["n2"], L["n3"], L["n4"])
    b.edge(L["n4"], L["n5"]); b.edge(L["n4"], L["n6"])
    b.edge(L["n5"], L["n7"]); b.edge(L["n6"], L["n7"])
    b.chain(L["n7"], L["n8"], L["n9"], L["n10"], L["n11"])
    b.chain(L["n12"], L["n13"], L["n14"], L["n15"], L["n16"])
    b.edge(L["n16"], L["n4"]); b.edge(L["n16"], L["n17"]); b.edge(L["n17"], L["x0"])
    # m1
    L["k1"] = b.fload(m1, t, p, F)
    L["k2"] = b.nop(m1)
    L["k3"] = b.new(m1, t, o2)
    L["k4"] = b.fstore(m1, p, F, t)
    L["k5"] = b.retv(m1, t)
    b.chain(L["e1"], L["k1"], L["k2"]); b.edge(L["k2"], L["k3"]); b.edge(L["k2"], L["k4"])
    b.chain(L["k3"], L["k4"], L["k5"], L["x1"])
    # m2
    L["j1"] = b.const(m2, u, o5)
    L["j2"] = b.retv(m2, u)
    b.chain(L["e2"], L["j1"], L["j2"], L["x2"])
    b.add_entry(m0)
    if m2_entry:
        b.add_entry(m2)
    g = b.build(name="tiny_m2" if m2_entry else "tiny")
    slots = {"x": 0, "y": 1, "z": 2, "a": 3, "R0": 4, "p": 5, "t": 6, "R1": 7, "u": 8, "R2": 9,
             "g": 10, "o1.f": 11, "o2.f": 12, "o3.ARR": 13}
    insts = {"N": 0, "o1": o1, "o2": o2, "o3": o3, "o4": o4, "o5": o5}
    return g, L, slots, insts


def tiny2():
    b = IcfgBuilder(n_fields=2)
    F = 1
    T = b.add_type([F])
    o1 = b.add_instance(T); o2 = b.add_instance(T); o3 = b.add_instance(T)
    g0 = b.add_static()
    dA = b.add_module(insts=[o1, o2], statics=[g0])
    dB = b.add_module(insts=[o1, o3], statics=[])
    m0 = b.add_method(dA, 0, 3)   # x y RET0
    m1 = b.add_method(dB, 1, 3)   # p t RET1
    x, y = b.L(m0, 0), b.L(m0, 1)
    p, t = b.L(m1, 0), b.L(m1, 1)
    L = {"e0": b.entry(m0), "x0": b.exit(m0), "e1": b.entry(m1), "x1": b.exit(m1)}
    L["s1"] = b.new(m0, x, o1)
    L["s2"] = b.new(m0, y, o2)
    L["s3"] = b.fstore(m0, x, F, y)
    L["s4"] = b.sstore(m0, b.S(g0), y)
    L["s5"], L["s6"] = b.call(m0, y, [x], [m1])
    L["s7"] = b.new(m1, t, o3)
    L["s8"] = b.fstore(m1, p, F, t)
    L["s9"] = b.retv(m1, t)
    b.chain(L["e0"], L["s1"], L["s2"], L["s3"], L["s4"], L["s5"])
    b.chain(L["s6"], L["x0"])
    b.chain(L["e1"], L["s7"], L["s8"], L["s9"], L["x1"])
    b.add_entry(m0)
    g = b.build(name="tiny2")
    slots = {"x": 0, "y": 1, "R0": 2, "p": 3, "t": 4, "R1": 5, "g": 6,
             "o1.f": 7, "o2.f": 8, "o3.f": 9}
    insts = {"N": 0, "o1": o1, "o2": o2, "o3": o3}
    return g, L, slots, insts


def tiny_args(wide_pad: int = 0):
    """A call with 5 parameters and one local passed three times (``r = m1(a, a, b, a, -)``),
    the shape whose wide-pool form lost parameters 4+ in round 1 (param_j <-
    arg_j for every j).  The callee stores through its first parameter, so a heap fact comes
    back through RET.  ``wide_pad`` > 0 pads the pool with field-less instances below and above
    the real ones (|Q| > 64: the wide-block path).  Expected sets: tiny_args.expected (by hand;
    the padding changes nothing)."""
    b = IcfgBuilder(n_fields=2)
    F = 1
    T = b.add_type([F]); T0 = b.add_type([])
    pad_lo = [b.add_instance(T0) for _ in range(wide_pad // 2)]
    o1 = b.add_instance(T); o2 = b.add_instance(T)
    pad_hi = [b.add_instance(T0) for _ in range(wide_pad - wide_pad // 2)]
    d = b.add_module(insts=pad_lo + [o1, o2] + pad_hi)
    m0 = b.add_method(d, 0, 4)    # a b r RET0
    m1 = b.add_method(d, 5, 7)    # p0 p1 p2 p3 p4 t RET1
    a, bb, r = (b.L(m0, i) for i in range(3))
    p0, p2, p3 = b.L(m1, 0), b.L(m1, 2), b.L(m1, 3)
    t = b.L(m1, 5)
    L = {"e0": b.entry(m0), "x0": b.exit(m0), "e1": b.entry(m1), "x1": b.exit(m1)}
    L["n1"] = b.new(m0, a, o1)
    L["n2"] = b.new(m0, bb, o2)
    L["n3"], L["n4"] = b.call(m0, r, [a, a, bb, a, -1], [m1])
    L["k0"] = b.fstore(m1, p0, F, p2)
    L["k1"] = b.copy(m1, t, p3)
    L["k2"] = b.retv(m1, t)
    b.chain(L["e0"], L["n1"], L["n2"], L["n3"])
    b.chain(L["n4"], L["x0"])
    b.chain(L["e1"], L["k0"], L["k1"], L["k2"], L["x1"])
    b.add_entry(m0)
    g = b.build(name=f"tiny_args{'_wide' if wide_pad else ''}")
    slots = {"a": 0, "b": 1, "r": 2, "R0": 3, "p0": 4, "p1": 5, "p2": 6, "p3": 7, "p4": 8,
             "t": 9, "R1": 10, "o1.f": 11, "o2.f": 12}
    insts = {"N": 0, "o1": o1, "o2": o2}
    return g, L, slots, insts


def fig2():
    b = IcfgBuilder(n_fields=1)
    T = b.add_type([])
    o = b.add_instance(T)
    d = b.add_module(insts=[o])
    m = b.add_method(d, 0, 2)     # x RET
    x = b.L(m, 0)
    L = {"entry": b.entry(m), "exit": b.exit(m)}
    for i in range(1, 7):
        L[f"L{i}"] = b.nop(m)
    L["L7"] = b.new(m, x, o)
    b.edge(L["entry"], L["L1"])
    b.edge(L["L1"], L["L2"]); b.edge(L["L1"], L["L4"])
    b.edge(L["L2"], L["L3"]); b.edge(L["L4"], L["L5"])
    b.edge(L["L3"], L["L6"]); b.edge(L["L5"], L["L6"])
    b.edge(L["L6"], L["L7"])
    b.edge(L["L7"], L["exit"]); b.edge(L["L7"], L["L1"])
    b.add_entry(m)
    return b.build(name="fig2"), L


def load_expected(name: str) -> Dict[str, set]:
    """Parse ``<name>.expected``: lines ``label: slot:inst slot:inst ...`` ('#' comments)."""
    out: Dict[str, set] = {}
    with open(os.path.join(HERE, name + ".expected")) as fh:
        for line in fh:
            line = line.split("#", 1)[0].strip()
            if not line:
                continue
            lab, rest = line.split(":", 1)
            facts = set()
            for tok in rest.split():
                s, o = tok.rsplit(":", 1)
                facts.add((s, o))
            out[lab.strip()] = facts
    return out
