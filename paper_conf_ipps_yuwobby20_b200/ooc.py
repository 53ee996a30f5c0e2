"""Out-of-core sub-graph streaming with dual buffering (§III-A1 "Dual-Buffering
Data Transfer").

When one app's fact store exceeds the device budget, "we have to divide the ICFG to sub-graphs
and process them in turn on GPU ... We allocate two buffers in the GPU memory and create two
CUDA execution streams ... The kernel engine keeps processing sub-graphs alternating between
the two buffers until the worklist algorithm converges".

B200 recast:
  * the ICFG is cut into K sub-graphs along method boundaries (contiguous method ranges with
    balanced node counts), so every INTRA and C2R edge stays inside one sub-graph and only
    CALL / RET edges cross;
  * sub-graph k is loaded as its own handle (tables resident, a few hundred bytes per node);
    its fact store lives in pinned host memory and is on the device only while k is solved:
    import (H2D) -> incremental build (keep_facts) -> export (D2H) -> release.  Two handles
    alternate on two CUDA streams, so the import of the next sub-graph overlaps the fixed
    point of the current one (the paper's dual buffering);
  * a crossing edge p -> s ends in a *proxy* of s inside p's sub-graph: a stub ENTRY of the
    callee (CALL) or a stub RETSITE (+ its CALL, for the V5 check) of the caller (RET).  Every
    method keeps its ENTRY/EXIT nodes in every sub-graph, so slot and instance gids are the
    global ones.  After a solve, each reached proxy's IN (= the union of T_e(OUT_p) over the
    crossing edges into it) is staged as a seed of the real node s in its own sub-graph
    (gdroid_stage_seeds: pairs OR-ed into IN(s), s queued — also with no pair, the first-reach
    rule A5);
  * sweeps over the sub-graphs repeat until no proxy delivers anything new.  IN only grows and
    every solve is a fair chaotic iteration of the same monotone equations, so the result is
    the least fixed point of the whole ICFG — checked against the oracle.
"""
from __future__ import annotations

import time
from dataclasses import dataclass, field
from types import SimpleNamespace
from typing import Dict, List, Optional

import numpy as np

E_INTRA, E_CALL, E_RET, E_C2R = range(4)
K_ENTRY, K_EXIT, K_RETSITE, K_CALL = 1, 2, 3, 4

_ARRAYS = ("row_ptr", "col", "edge_kind", "node_kind", "node_method", "node_ops", "call_arg_ptr",
           "call_args", "method_entry", "method_exit", "method_module", "method_n_locals",
           "method_n_params", "module_inst_ptr", "module_insts", "module_static_ptr",
           "module_statics", "inst_type", "type_field_ptr", "type_fields", "entries")


def partition_methods(g, n_parts: int) -> np.ndarray:
    """part[m] for every method: contiguous method ranges with about equal node counts."""
    M = len(g.method_entry)
    per = np.bincount(g.node_method.astype(np.int64), minlength=M)
    cum = np.cumsum(per)
    tot = int(cum[-1]) if M else 0
    part = np.minimum((cum - per) * n_parts // max(tot, 1), n_parts - 1).astype(np.int64)
    return part


@dataclass
class SubGraph:
    icfg: object                      # duck-typed gdroid_icfg_desc arrays (see _binding.make_desc)
    glob: np.ndarray                  # sub node id -> global node id
    owned: np.ndarray                 # sub node is a real node of this sub-graph
    proxies: np.ndarray               # sub node ids of proxies (stub ENTRY / RETSITE of other parts)
    proxy_glob: np.ndarray            # global node id each proxy stands for
    sub_of: Dict[int, int] = field(default_factory=dict)   # global -> sub id (owned nodes)


def make_subgraph(g, part: np.ndarray, k: int) -> SubGraph:
    """Sub-graph k: its methods' nodes, plus ENTRY/EXIT stubs of every other method and stub
    RETSITE/CALL pairs of other parts' call sites that its exits return to."""
    N = len(g.node_kind)
    rp = g.row_ptr.astype(np.int64)
    nm = g.node_method.astype(np.int64)
    own = part[nm] == k
    keep = own.copy()
    keep[g.method_entry] = True
    keep[g.method_exit] = True
    ops = g.node_ops.reshape(-1, 4)
    # RET edges from owned exits to retsites of other parts: stub the RETSITE and its CALL
    src = np.repeat(np.arange(N), np.diff(rp))
    ek = g.edge_kind
    ret = (ek == E_RET) & own[src] & ~own[g.col]
    stub_rs = np.unique(g.col[ret])
    keep[stub_rs] = True
    stub_calls = ops[stub_rs, 3].astype(np.int64)
    keep[stub_calls] = True
    glob = np.nonzero(keep)[0]
    sub = -np.ones(N, dtype=np.int64)
    sub[glob] = np.arange(len(glob))
    stub_call_mask = np.zeros(N, dtype=bool)
    stub_call_mask[stub_calls] = True
    # edges: every out-edge of an owned node; stub CALLs keep C2R and CALL edges (V5 checks)
    e_keep = own[src] | (stub_call_mask[src] & ~own[src] & ((ek == E_C2R) | (ek == E_CALL)))
    es, ed, ekk = src[e_keep], g.col[e_keep], ek[e_keep]
    assert (sub[ed] >= 0).all()
    order = np.argsort(sub[es], kind="stable")
    es, ed, ekk = es[order], ed[order], ekk[order]
    n_sub = len(glob)
    row_ptr = np.zeros(n_sub + 1, dtype=np.uint64)
    np.cumsum(np.bincount(sub[es], minlength=n_sub), out=row_ptr[1:])
    new_ops = ops[glob].copy()
    rs = g.node_kind[glob] == K_RETSITE
    new_ops[rs, 3] = sub[new_ops[rs, 3]]
    # call args for kept CALL nodes
    ap = g.call_arg_ptr.astype(np.int64)
    cnt = np.diff(ap)[glob]
    is_call = g.node_kind[glob] == K_CALL
    cnt = np.where(is_call, cnt, 0)
    arg_ptr = np.zeros(n_sub + 1, dtype=np.uint64)
    np.cumsum(cnt, out=arg_ptr[1:])
    idx = np.concatenate([np.arange(ap[n], ap[n + 1]) for n in glob[is_call]]) if is_call.any() else np.zeros(0, np.int64)
    args = g.call_args[idx.astype(np.int64)] if len(idx) else np.zeros(0, np.int32)
    ent = [int(sub[e]) for e in g.entries if own[e]]
    d = {nm_: getattr(g, nm_) for nm_ in _ARRAYS}
    d.update(row_ptr=row_ptr, col=sub[ed].astype(np.uint32), edge_kind=ekk.astype(np.uint8),
             node_kind=g.node_kind[glob].copy(), node_method=g.node_method[glob].copy(),
             node_ops=new_ops.reshape(-1).astype(np.int32), call_arg_ptr=arg_ptr,
             call_args=np.asarray(args, dtype=np.int32),
             method_entry=sub[g.method_entry].astype(np.uint32), method_exit=sub[g.method_exit].astype(np.uint32),
             entries=np.asarray(ent, dtype=np.uint32))
    ic = SimpleNamespace(**d)
    ic.n_nodes, ic.n_edges, ic.n_entries = n_sub, int(row_ptr[-1]), len(ent)
    for a in ("n_methods", "n_modules", "n_types", "n_instances", "n_statics", "n_fields"):
        setattr(ic, a, getattr(g, a))
    ic.nbytes = lambda: sum(np.asarray(getattr(ic, x)).nbytes for x in _ARRAYS)
    owned = own[glob]
    nk = g.node_kind[glob]
    # proxies: stub ENTRYs of other parts' methods, stub RETSITEs
    prox = np.nonzero(~owned & ((nk == K_ENTRY) | (nk == K_RETSITE)))[0]
    return SubGraph(ic, glob, owned, prox, glob[prox],
                    {int(gid): int(i) for i, gid in enumerate(glob) if owned[i]})


@dataclass
class OocStats:
    sweeps: int = 0
    solves: int = 0
    rounds: int = 0
    visits: int = 0
    h2d_bytes: int = 0
    d2h_bytes: int = 0
    seeds: int = 0
    seconds: float = 0.0
    build_ms: float = 0.0
    peak_resident_fact_bytes: int = 0


class OutOfCore:
    """Solve one app's IDFG with at most two sub-graph fact stores on the device."""

    def __init__(self, g, n_parts: int, device: int = 0):
        import torch
        from . import _binding as gd
        self.g, self.K, self.device = g, n_parts, device
        self.part = partition_methods(g, n_parts)
        self.subs = [make_subgraph(g, self.part, k) for k in range(n_parts)]
        self.streams = [torch.cuda.Stream(device=device), torch.cuda.Stream(device=device)]
        self.handles = []
        self.host = []                                    # pinned fact stores (the "home" copies)
        self._pin = []
        for k, sg in enumerate(self.subs):
            h = gd.load(sg.icfg, device=device, stream=self.streams[k % 2].cuda_stream)
            h.release_facts()
            t = torch.zeros(h.fact_bytes // 8, dtype=torch.int64, pin_memory=True)
            self._pin.append(t)
            self.host.append(t.numpy().view(np.uint64))
            self.handles.append(h)
        self.owner_sub = {}                               # global node -> (part, sub id) of owned nodes
        for k, sg in enumerate(self.subs):
            for gid, si in sg.sub_of.items():
                self.owner_sub[gid] = (k, si)
        self.stats = OocStats()

    def run(self, max_sweeps: int = 10_000) -> OocStats:
        """Sweeps over the sub-graphs until no proxy delivers new facts or a new first reach."""
        K, st = self.K, self.stats
        t0 = time.perf_counter()
        pending: List[Dict[int, set]] = [dict() for _ in range(K)]      # sub id -> pairs to seed
        sent: List[Dict[int, set]] = [dict() for _ in range(K)]         # per part: proxy -> delivered
        fresh = [True] * K
        for sweep in range(max_sweeps):
            todo = [k for k in range(K) if fresh[k] or pending[k]]
            if not todo:
                break
            st.sweeps += 1
            self.handles[todo[0]].import_facts(self.host[todo[0]])
            for idx, k in enumerate(todo):
                h, sg = self.handles[k], self.subs[k]
                if pending[k]:
                    nodes = np.array(sorted(pending[k]), dtype=np.uint32)
                    lists = [np.array(sorted(pending[k][n]), dtype=np.uint64) for n in nodes]
                    ptr = np.zeros(len(nodes) + 1, dtype=np.uint64)
                    np.cumsum([len(x) for x in lists], out=ptr[1:])
                    pairs = np.concatenate(lists) if lists else np.zeros(0, np.uint64)
                    h.stage_seeds(nodes, ptr, pairs)
                    st.seeds += len(pairs)
                    pending[k] = {}
                h.build(keep_facts=True, asynchronous=True)
                st.h2d_bytes += h.fact_bytes
                if idx + 1 < len(todo):                   # dual buffering: next import overlaps
                    nk = todo[idx + 1]
                    self.handles[nk].import_facts(self.host[nk])
                    st.peak_resident_fact_bytes = max(st.peak_resident_fact_bytes,
                                                      h.fact_bytes + self.handles[nk].fact_bytes)
                s = h.sync()
                fresh[k] = False
                st.solves += 1
                st.rounds += s["rounds"]
                st.visits += s["node_visits"]
                st.build_ms += s["build_ns"] / 1e6
                # boundary: reached proxies deliver IN(proxy) to the real node's sub-graph
                if len(sg.proxies):
                    reached = h.read_reached(sg.proxies)
                    ptr, pairs = h.read_nodes_facts(sg.proxies)
                    for i, (p, gid) in enumerate(zip(sg.proxies.tolist(), sg.proxy_glob.tolist())):
                        if not reached[i]:
                            continue
                        have = set(pairs[int(ptr[i]):int(ptr[i + 1])].tolist())
                        prev = sent[k].get(p)
                        if prev is not None and have <= prev:
                            continue
                        new = have - (prev or set())
                        sent[k][p] = have | (prev or set())
                        tk, ts = self.owner_sub[gid]
                        pending[tk].setdefault(ts, set()).update(new)
                h.export_facts(self.host[k])
                st.d2h_bytes += h.fact_bytes
                h.release_facts()                         # stream-ordered after the export
            for h in self.handles:
                h.stream_sync()
        st.seconds = time.perf_counter() - t0
        return st

    def read_all_facts(self):
        """(ptr[N+1], pairs) over the ORIGINAL node ids: each owned node from its sub-graph."""
        N = len(self.g.node_kind)
        per = [None] * N
        for k, (h, sg) in enumerate(zip(self.handles, self.subs)):
            h.import_facts(self.host[k])
            h.build(keep_facts=True)                      # nothing staged: an empty round
            ptr, pairs = h.read_all_facts()
            for si in np.nonzero(sg.owned)[0].tolist():
                per[int(sg.glob[si])] = pairs[int(ptr[si]):int(ptr[si + 1])]
            h.release_facts()
        out_ptr = np.zeros(N + 1, dtype=np.uint64)
        np.cumsum([len(x) for x in per], out=out_ptr[1:])
        return out_ptr, (np.concatenate(per) if N else np.zeros(0, np.uint64))

    def free(self):
        for h in self.handles:
            h.free()
        self.handles = []
