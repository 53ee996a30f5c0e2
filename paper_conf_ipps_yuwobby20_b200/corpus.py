"""Multi-GPU corpus driver: apps are sharded across ranks, never a single ICFG.

One process per GPU (torchrun).  Every app's IDFG is an independent fixed point (Eq. 1,
PAPER.md:351-355), so there is no data-path collective: each rank builds its shard with the
C-ABI library (batched apps share device rounds) and the ranks only exchange one fixed-size
record each at the end (NCCL over NVLink on GPUs; gloo in the CPU tests).

Host-side pieces here are plain Python and are tested on CPU (tests/test_corpus_host.py):
LPT sharding, batching under a node budget, record packing and the gather.
"""
from __future__ import annotations

import threading
import time
from dataclasses import dataclass, field
from queue import Queue
from typing import Callable, Dict, List, Optional, Sequence

import numpy as np

RECORD_FIELDS = ("apps", "visits", "alg_bytes", "build_ns", "wall_ns", "max_app_ns",
                 "digest_sum", "errors")


def lpt_shard(sizes: Sequence[int], world: int, per_rank: Optional[int] = None) -> List[List[int]]:
    """Longest-processing-time-first assignment of apps (estimated cost = size) to ranks.
    With per_rank set, every rank gets exactly that many apps (weak scaling)."""
    order = sorted(range(len(sizes)), key=lambda i: (-sizes[i], i))
    loads = [0] * world
    shard: List[List[int]] = [[] for _ in range(world)]
    for i in order:
        cands = [r for r in range(world) if per_rank is None or len(shard[r]) < per_rank]
        r = min(cands, key=lambda q: (loads[q], q))
        shard[r].append(i)
        loads[r] += sizes[i]
    return [sorted(s) for s in shard]


def batches_under_budget(app_ids: Sequence[int], sizes: Sequence[int], node_budget: int) -> List[List[int]]:
    """Group a rank's apps into batches of at most node_budget estimated nodes (an app larger
    than the budget forms its own batch).  Apps in a batch share every device round."""
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


def gather_records(rec: np.ndarray, device=None) -> np.ndarray:
    """all_gather of one record per rank over the default process group (NCCL or gloo)."""
    import torch
    import torch.distributed as dist
    t = torch.from_numpy(np.ascontiguousarray(rec)).to(device if device is not None else "cpu")
    if not dist.is_available() or not dist.is_initialized():
        return t.cpu().numpy().reshape(1, -1)
    bufs = [torch.zeros_like(t) for _ in range(dist.get_world_size())]
    dist.all_gather(bufs, t)
    return torch.stack(bufs).cpu().numpy()


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


@dataclass
class BatchResult:
    app_ids: List[int]
    digests: np.ndarray
    stats: dict
    ms: float


def run_shard(app_ids: Sequence[int], make_app: Callable[[int], object], sizes: Sequence[int],
              device: int = 0, stream: int = 0, node_budget: int = 4_000_000,
              prefetch: bool = True) -> List[BatchResult]:
    """Build every app of this rank's shard on `device`, batch by batch.  A loader thread
    generates the next batch and uploads it (gdroid_load_batch on its own stream) while the GPU
    builds the current one — the paper's dual-buffered transfer."""
    import torch
    from . import _binding as gd
    plan = batches_under_budget(app_ids, sizes, node_budget)
    q: "Queue" = Queue(maxsize=1 if prefetch else 0)
    streams = [torch.cuda.Stream(device=device), torch.cuda.Stream(device=device)]

    def loader():
        for j, b in enumerate(plan):
            apps = [make_app(i) for i in b]
            t0 = time.perf_counter()
            h = gd.load(apps, device=device, stream=streams[j % 2].cuda_stream)
            q.put((b, h, (time.perf_counter() - t0) * 1e3))
        q.put(None)

    th = threading.Thread(target=loader, daemon=True)
    th.start()
    out: List[BatchResult] = []
    while True:
        item = q.get()
        if item is None:
            break
        ids, app, load_ms = item
        t0 = time.perf_counter()
        st = app.build()
        dig = app.app_digests()
        app.free()
        out.append(BatchResult(list(ids), dig, st, (time.perf_counter() - t0) * 1e3 + load_ms))
    th.join()
    return out
