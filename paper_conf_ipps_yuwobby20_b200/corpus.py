"""Multi-GPU corpus driver: apps are sharded across ranks, never a single ICFG.

One process per GPU (torchrun).  Every app's IDFG is an independent fixed point (Eq. 1,
PAPER.md:351-355), so there is no data-path collective: each rank builds its shard with the
C-ABI library (apps of a batch share device rounds) and the ranks exchange, at the end, one
fixed int64[8] record each plus the per-app digests (NCCL over NVLink on GPUs; gloo in the
CPU tests).  This module is the ONE multi-GPU path: bench.py and the tests call it.

Pieces:
  * plan_corpus       LPT sharding of the apps over ranks by estimated cost (narrow and wide
                      apps weighted by their measured per-node cost), then per-rank batches
                      (narrow apps under a node budget, wide apps alone or in small groups).
  * DeviceShard       device-resident rank state: every batch's tables loaded once; a batch
                      holds a fact store only while it builds (gdroid_build_opts.release_facts),
                      so a 1000-app shard fits one B200.
  * run_rank          warm-up + timed steps over a shard object (DeviceShard, or a CPU stub in
                      the tests), bracketed by barriers; the device clock is supplied by the
                      caller.
  * gather_records / gather_digests / check_digests
                      the end-of-run exchange and rank 0's comparison with the oracle cache.
  * run_pipelined     the end-to-end path: a loader thread generates and uploads batch i+1
                      (gdroid_load_batch on its own stream, the paper's dual buffering,
                      PAPER.md:544-580) while batch i builds and its facts are read back.
"""
from __future__ import annotations

import threading
import time
from concurrent.futures import ThreadPoolExecutor
from dataclasses import dataclass, field
from queue import Queue
from typing import Callable, Dict, List, Optional, Sequence

import numpy as np

RECORD_FIELDS = ("apps", "visits", "alg_bytes", "build_ns", "wall_ns", "max_app_ns",
                 "digest_sum", "errors")

# Per-node device cost of a wide app (|Q| = 256: 4 words per row, row-occupancy path)
# relative to a narrow one, measured in round 1 (worst 221 ms / 1.92M nodes
# vs the 8-app narrow shard 23.7 ms / 2.03M nodes, ~9.9x).  Only the LPT weights use it.
WIDE_COST = 10.0


# ---------------------------------------------------------------------------------- planning
def lpt_shard(costs: Sequence[float], world: int, per_rank: Optional[int] = None) -> List[List[int]]:
    """Longest-processing-time-first assignment of apps to ranks by estimated cost.
    With per_rank set, every rank gets exactly that many apps (weak scaling)."""
    order = sorted(range(len(costs)), key=lambda i: (-costs[i], i))
    loads = [0.0] * world
    shard: List[List[int]] = [[] for _ in range(world)]
    for i in order:
        cands = [r for r in range(world) if per_rank is None or len(shard[r]) < per_rank]
        r = min(cands, key=lambda q: (loads[q], q))
        shard[r].append(i)
        loads[r] += costs[i]
    return [sorted(s) for s in shard]


def batches_under_budget(app_ids: Sequence[int], sizes: Sequence[int], node_budget: int) -> List[List[int]]:
    """Group apps into batches of at most node_budget estimated nodes (an app larger than the
    budget forms its own batch).  Apps in a batch share every device round."""
    out: List[List[int]] = []
    cur: List[int] = []
    acc = 0
    for i in app_ids:
        if cur and acc + sizes[i] > node_budget:
            out.append(cur)
            cur, acc = [], 0
        cur.append(i)
        acc += sizes[i]
    if cur:
        out.append(cur)
    return out


@dataclass
class Plan:
    n_apps: int
    world: int
    sizes: List[int]                       # estimated nodes per app
    wide: List[bool]                       # |Q| > 64 (worst-case shape)
    shards: List[List[int]]                # app ids per rank
    batches: List[List[List[int]]]         # per rank: batches of app ids

    def cost(self, i: int) -> float:
        return self.sizes[i] * (WIDE_COST if self.wide[i] else 1.0)


def plan_corpus(sizes: Sequence[int], wide: Sequence[bool], world: int, node_budget: int = 4_000_000,
                wide_per_batch: int = 1, per_rank: Optional[int] = None,
                app_ids: Optional[Sequence[int]] = None) -> Plan:
    """LPT over ranks by cost, then per rank: wide apps in groups of wide_per_batch (their
    fact stores are ~35 GB each), narrow apps in id order under node_budget."""
    ids = list(range(len(sizes))) if app_ids is None else list(app_ids)
    costs_sub = [sizes[i] * (WIDE_COST if wide[i] else 1.0) for i in ids]
    shards = [[ids[j] for j in s] for s in lpt_shard(costs_sub, world, per_rank)]
    batches = []
    for s in shards:
        w = [i for i in s if wide[i]]
        n = [i for i in s if not wide[i]]
        bw = [w[k:k + wide_per_batch] for k in range(0, len(w), max(1, wide_per_batch))]
        batches.append(bw + batches_under_budget(n, sizes, node_budget))
    return Plan(len(sizes), world, list(sizes), list(wide), [sorted(s) for s in shards], batches)


def make_apps(ids: Sequence[int], make_app: Callable[[int], object], threads: int = 8) -> Dict[int, object]:
    """Generate apps in a thread pool (the C++ generator releases the GIL)."""
    with ThreadPoolExecutor(max_workers=max(1, threads)) as ex:
        return dict(zip(ids, ex.map(make_app, ids)))


# ---------------------------------------------------------------------------------- records
def pack_record(**kw) -> np.ndarray:
    """Fixed int64[8] per-rank record; unknown keys are rejected."""
    bad = set(kw) - set(RECORD_FIELDS)
    if bad:
        raise KeyError(f"unknown record fields {sorted(bad)}")
    rec = np.zeros(len(RECORD_FIELDS), dtype=np.int64)
    for k, v in kw.items():
        rec[RECORD_FIELDS.index(k)] = np.int64(np.uint64(int(v) & 0xFFFFFFFFFFFFFFFF).view(np.int64))
    return rec


def unpack_records(recs: np.ndarray) -> List[Dict[str, int]]:
    out = []
    for row in np.asarray(recs).reshape(-1, len(RECORD_FIELDS)):
        d = {k: int(v) for k, v in zip(RECORD_FIELDS, row)}
        d["digest_sum"] &= 0xFFFFFFFFFFFFFFFF
        out.append(d)
    return out


def _all_gather(t, device):
    import torch
    import torch.distributed as dist
    t = t.to(device) if device is not None else t
    if not dist.is_available() or not dist.is_initialized():
        return t.cpu().unsqueeze(0)
    bufs = [torch.zeros_like(t) for _ in range(dist.get_world_size())]
    dist.all_gather(bufs, t)
    return torch.stack(bufs).cpu()


def gather_records(rec: np.ndarray, device=None) -> np.ndarray:
    """all_gather of one record per rank over the default process group (NCCL or gloo)."""
    import torch
    return _all_gather(torch.from_numpy(np.ascontiguousarray(rec)), device).numpy().reshape(-1, len(RECORD_FIELDS))


def gather_digests(n_apps: int, digests: Dict[int, int], device=None):
    """Every rank contributes its apps' digests at their corpus index (others 0); the gather
    gives each app's digest from the one rank that built it: (uint64[n_apps], count[n_apps])."""
    import torch
    v = np.zeros(n_apps, dtype=np.uint64)
    m = np.zeros(n_apps, dtype=np.int64)
    for i, d in digests.items():
        v[i] = np.uint64(int(d) & 0xFFFFFFFFFFFFFFFF)
        m[i] = 1
    t = torch.from_numpy(np.concatenate([v.view(np.int64), m]))
    g = _all_gather(t, device).numpy()
    vals, masks = g[:, :n_apps].view(np.uint64), g[:, n_apps:]
    if (masks.sum(0) > 1).any():
        raise RuntimeError("an app was built by more than one rank")
    out = np.zeros(n_apps, dtype=np.uint64)
    for r in range(g.shape[0]):
        out[masks[r] == 1] = vals[r][masks[r] == 1]
    return out, masks.sum(0)


def check_digests(digests: np.ndarray, mask: np.ndarray, cache: Dict[str, dict]) -> dict:
    """Compare the gathered per-app digests with the oracle cache (tests/golden/
    corpus_digests.json, written by scripts/make_corpus_digests.py from oracle/ alone)."""
    checked, bad, missing = 0, [], 0
    for i in np.nonzero(mask)[0].tolist():
        ref = cache.get(str(i))
        if ref is None:
            missing += 1
            continue
        checked += 1
        if str(int(digests[i])) != ref["app_digest"]:
            bad.append(i)
    return {"checked": checked, "mismatches": bad, "not_in_cache": missing}


def combine(records: List[Dict[str, int]]) -> Dict[str, int]:
    tot = {k: 0 for k in RECORD_FIELDS}
    for r in records:
        for k in RECORD_FIELDS:
            if k in ("wall_ns", "max_app_ns"):
                tot[k] = max(tot[k], r[k])
            elif k == "digest_sum":
                tot[k] = (tot[k] + r[k]) & 0xFFFFFFFFFFFFFFFF
            else:
                tot[k] += r[k]
    return tot


# ---------------------------------------------------------------------------------- device shard
class DeviceShard:
    """One rank's batches, tables resident on the device; the fact store of a batch exists only
    while it builds (release_facts), drawn from the device's stream-ordered pool."""

    def __init__(self, batches: List[List[int]], apps: Dict[int, object], device: int = 0, stream: int = 0):
        from . import _binding as gd
        self.batches = batches
        self.handles = []
        self.nodes = []
        self.input_bytes = 0
        for b in batches:
            h = gd.load([apps[i] for i in b], device=device, stream=stream)
            h.release_facts()                              # tables stay, facts only while building
            self.handles.append(h)
            self.nodes.append(sum(apps[i].n_nodes for i in b))
            self.input_bytes += sum(apps[i].nbytes() for i in b)
        self.stats: List[dict] = []

    def step(self, byte_model: bool = False) -> None:
        """Enqueue one build of every batch (asynchronous; the device runs them back to back)."""
        for h in self.handles:
            h.build(asynchronous=True, byte_model=byte_model, release_facts=True)

    def finish(self) -> List[dict]:
        self.stats = [h.sync() for h in self.handles]
        return self.stats

    def digests(self) -> Dict[int, int]:
        out = {}
        for b, h in zip(self.batches, self.handles):
            for k, i in enumerate(b):
                out[i] = int(h.app_digests()[k])
        return out

    def free(self):
        for h in self.handles:
            h.free()
        self.handles = []


@dataclass
class RankResult:
    step_ms: List[float]
    stats: List[dict]
    digests: Dict[int, int]
    counted: Optional[List[dict]] = None


def run_rank(shard, steps: int, warmup: int, barrier: Callable[[], None],
             timer: Callable[[Callable[[], None]], float], count_bytes: bool = True) -> RankResult:
    """W untimed steps, then K timed steps bracketed by barriers; `timer(fn)` runs fn and
    returns its device-clock milliseconds (CUDA events on the launching stream).  One extra,
    untimed step with the counting kernel instantiation gives the byte models."""
    for _ in range(warmup):
        shard.step()
        shard.finish()
    barrier()

    def timed():
        for _ in range(steps):                              # one build per batch per step
            shard.step()
            shard.finish()

    ms = timer(timed)
    stats = list(shard.stats)
    digests = shard.digests()
    barrier()
    counted = None
    if count_bytes:
        shard.step(byte_model=True)
        counted = shard.finish()
        if shard.digests() != digests:
            raise RuntimeError("the counting build gave other digests")
    return RankResult([ms], stats, digests, counted)


# ---------------------------------------------------------------------------------- end to end
@dataclass
class BatchResult:
    app_ids: List[int]
    digests: np.ndarray
    stats: dict
    ms: float
    d2h_bytes: int = 0
    h2d_bytes: int = 0


class PinnedBuf:
    """Growable pinned host buffer (uint64) for fact readback; reused across batches and steps
    (pinning is slow, so an untimed warm-up pass sizes it)."""

    def __init__(self):
        self.t = None

    def get(self, n: int) -> np.ndarray:
        import torch
        if self.t is None or self.t.numel() < n:
            self.t = None
            self.t = torch.empty(max(int(n * 1.1), 1 << 20), dtype=torch.int64, pin_memory=True)
        return self.t.numpy().view(np.uint64)[:n]


class ReadbackBuffers:
    def __init__(self):
        self.ptr, self.pairs, self.total = PinnedBuf(), PinnedBuf(), PinnedBuf()
        self.cap = 0                                  # pairs capacity the async readback may use


def run_pipelined(batches: List[List[int]], make_app: Callable[[int], object], device: int = 0,
                  readback: str = "facts", on_facts: Optional[Callable] = None,
                  bufs: Optional[ReadbackBuffers] = None, reserve_sms: int = 0) -> List[BatchResult]:
    """End to end through the public API: a loader thread generates batch i+1 and uploads it
    (gdroid_load_batch on its own stream: the paper's dual buffering) while
    batch i builds.  As soon as batch i's fixed point is done its facts are expanded on the device
    and their copy to pinned host memory is enqueued (gdroid_read_batch_facts_async — Alg. 3
    l.17 h_fact <- d_fact); batch i+1's fixed point then runs while the copy engine
    moves batch i's facts.  readback='digests' reads only the app digests.  A loader failure is
    re-raised here."""
    import torch
    from . import _binding as gd
    q: "Queue" = Queue(maxsize=1)
    streams = [torch.cuda.Stream(device=device), torch.cuda.Stream(device=device)]
    stop = threading.Event()
    bufs = bufs or ReadbackBuffers()
    facts = readback == "facts"

    def loader():
        try:
            for j, b in enumerate(batches):
                if stop.is_set():
                    break
                apps = [make_app(i) for i in b]
                t0 = time.perf_counter()
                h = gd.load(apps, device=device, stream=streams[j % 2].cuda_stream)
                h.release_facts()          # the build allocates it: two fact stores live, not three
                q.put((b, h, (time.perf_counter() - t0) * 1e3, [a.n_nodes for a in apps],
                       sum(a.nbytes() for a in apps)))
        except BaseException as e:                         # surface it in the consumer
            q.put(e)
        finally:
            q.put(None)

    out: List[BatchResult] = []

    pending = {"async": False}

    def start_readback(cur):
        ids, app, st, t0, load_ms, nn = cur[:6]
        pending["async"] = False
        if facts and bufs.cap:
            n = sum(nn)
            pending["async"] = app.read_batch_facts_async(bufs.ptr.get(n + 1), bufs.pairs.get(bufs.cap),
                                                          bufs.total.get(1))

    def finish(prev):
        ids, app, st, t0, load_ms, nn, ib = prev
        dig = app.app_digests()
        d2h = 8 * len(ids)
        if facts:
            n = sum(nn)
            app.stream_sync()                              # the async readback (if any) is done
            tot = int(bufs.total.get(1)[0]) if pending["async"] else -1
            if 0 <= tot <= bufs.cap:
                ptr, pairs = bufs.ptr.get(n + 1), bufs.pairs.get(bufs.cap)[:tot]
            else:                                          # first pass / too small: synchronous, grow
                ptr, pairs = app.read_batch_facts(bufs.ptr, bufs.pairs)
                bufs.cap = max(bufs.cap, int(1.25 * len(pairs)) + (1 << 20))
            d2h += ptr.nbytes + pairs.nbytes
            if on_facts is not None:
                base = 0
                for k, i in enumerate(ids):
                    p = ptr[base:base + nn[k] + 1]
                    on_facts(i, p - p[0], pairs[int(p[0]):int(p[-1])])
                    base += nn[k]
        app.free()
        out.append(BatchResult(list(ids), dig, st, (time.perf_counter() - t0) * 1e3 + load_ms, d2h, ib))

    th = threading.Thread(target=loader, daemon=True)
    th.start()
    prev = None
    try:
        while True:
            item = q.get()
            if item is None:
                break
            if isinstance(item, BaseException):
                raise item
            ids, app, load_ms, nn, ib = item
            t0 = time.perf_counter()
            app.build(asynchronous=True, reserve_sms=reserve_sms if facts else 0)
            if prev is not None:                          # batch i-1's readback ran beside it
                finish(prev)
                prev = None
            st = app.sync()
            prev = (ids, app, st, t0, load_ms, nn, ib)
            start_readback(prev)
        if prev is not None:
            finish(prev)
            prev = None
    finally:
        stop.set()
        if prev is not None:
            prev[1].stream_sync()
            prev[1].free()
        while th.is_alive() or not q.empty():             # drain so the loader can finish
            try:
                it = q.get(timeout=0.1)
                if isinstance(it, tuple):
                    it[1].free()
            except Exception:
                if not th.is_alive():
                    break
        th.join()
    return out


def run_shard(app_ids: Sequence[int], make_app: Callable[[int], object], sizes: Sequence[int],
              device: int = 0, stream: int = 0, node_budget: int = 4_000_000,
              prefetch: bool = True, readback: str = "digests") -> List[BatchResult]:
    """Build every app of a shard batch by batch through run_pipelined (kept for callers of
    the round-1 API)."""
    return run_pipelined(batches_under_budget(app_ids, sizes, node_budget), make_app, device=device,
                         readback=readback)
