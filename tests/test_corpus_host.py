"""Host logic of the multi-GPU corpus driver (CPU, gloo world_size 2): sharding, batching,
record packing and the all_gather of per-rank records."""
from __future__ import annotations

import os
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp

from paper_conf_ipps_yuwobby20_b200 import corpus
from synth import generator as G


def test_plan_corpus_1000_strong():
    """The bench's corpus1000 plan: every app on exactly one rank, wide (|Q| = 256) apps in
    their own batches, narrow batches under the node budget, LPT cost balance."""
    n = 1000
    sizes = G.corpus_sizes(n)
    wide = [G.corpus_config(i).q_cap > 64 for i in range(n)]
    assert sum(wide) == 15
    for world in (1, 2, 4, 8):
        p = corpus.plan_corpus(sizes, wide, world, node_budget=4_000_000)
        flat = sorted(i for s in p.shards for i in s)
        assert flat == list(range(n))
        assert sorted(i for bs in p.batches for b in bs for i in b) == flat
        for bs in p.batches:
            for b in bs:
                if any(wide[i] for i in b):
                    assert len(b) == 1
                else:
                    assert len(b) == 1 or sum(sizes[i] for i in b) <= 4_000_000
        loads = [sum(p.cost(i) for i in s) for s in p.shards]
        assert max(loads) - min(loads) <= max(p.cost(i) for i in range(n))


def test_lpt_shard_balanced_and_exact():
    sizes = G.corpus_sizes(64)
    for world in (1, 2, 4, 8):
        sh = corpus.lpt_shard(sizes, world, per_rank=64 // world)
        flat = sorted(i for s in sh for i in s)
        assert flat == list(range(64))                      # every app exactly once
        assert all(len(s) == 64 // world for s in sh)       # weak scaling: fixed per rank
        loads = [sum(sizes[i] for i in s) for s in sh]
        assert max(loads) <= 1.6 * (sum(loads) / world) + max(sizes)
    free = corpus.lpt_shard(sizes, 3)
    loads = [sum(sizes[i] for i in s) for s in free]
    assert max(loads) - min(loads) <= max(sizes)            # LPT bound


def test_batches_under_budget():
    sizes = [5, 5, 5, 20, 1, 1]
    b = corpus.batches_under_budget(range(6), sizes, 10)
    assert b == [[0, 1], [2], [3], [4, 5]]
    assert sorted(i for x in b for i in x) == list(range(6))


def test_record_roundtrip():
    r = corpus.pack_record(apps=3, visits=10, digest_sum=(1 << 64) - 5, wall_ns=7)
    d = corpus.unpack_records(r)[0]
    assert d["apps"] == 3 and d["digest_sum"] == (1 << 64) - 5 and d["wall_ns"] == 7
    with pytest.raises(KeyError):
        corpus.pack_record(bogus=1)
    tot = corpus.combine([d, d])
    assert tot["apps"] == 6 and tot["wall_ns"] == 7 and tot["digest_sum"] == ((1 << 65) - 10) % (1 << 64)


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, out):
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    sizes = G.corpus_sizes(16)
    shard = corpus.lpt_shard(sizes, world, per_rank=16 // world)[rank]
    rec = corpus.pack_record(apps=len(shard), visits=sum(shard), digest_sum=rank + 1,
                             wall_ns=100 * (rank + 1))
    recs = corpus.gather_records(rec)
    out.put((rank, recs.tolist(), shard))
    dist.destroy_process_group()


def test_gather_over_gloo_world2():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in ps:
        p.start()
    res = [q.get(timeout=120) for _ in range(2)]
    for p in ps:
        p.join(timeout=60)
        assert p.exitcode == 0
    res.sort()
    shards = [r[2] for r in res]
    assert sorted(shards[0] + shards[1]) == list(range(16))
    for _, recs, _ in res:                                  # every rank sees both records
        tot = corpus.combine(corpus.unpack_records(np.array(recs)))
        assert tot["apps"] == 16 and tot["digest_sum"] == 3 and tot["wall_ns"] == 200
        assert tot["visits"] == sum(range(16))


class _StubShard:
    """CPU stand-in for corpus.DeviceShard: 'builds' return a fixed digest per app."""

    def __init__(self, batches, digest_of):
        self.batches, self.digest_of, self.stats, self.built = batches, digest_of, [], 0

    def step(self, byte_model=False):
        self.built += 1

    def finish(self):
        self.stats = [{"node_visits": len(b), "fixpoint_ns": 1, "alg_bytes": 8, "build_ns": 2}
                      for b in self.batches]
        return self.stats

    def digests(self):
        return {i: self.digest_of(i) for b in self.batches for i in b}


def _rank_path_worker(rank, world, port, out):
    """bench.py's corpus path on one rank with the build stubbed: plan, run_rank (barriers),
    record + digest gathers, rank 0's check against a digest cache."""
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    n = 40
    sizes = G.corpus_sizes(n)
    wide = [G.corpus_config(i).q_cap > 64 for i in range(n)]
    plan = corpus.plan_corpus(sizes, wide, world, node_budget=1_000_000)
    dig = lambda i: (i * 0x9E3779B97F4A7C15 + 7) & ((1 << 64) - 1)
    shard = _StubShard(plan.batches[rank], dig)
    res = corpus.run_rank(shard, steps=3, warmup=2, barrier=dist.barrier, timer=lambda fn: (fn(), 5.0)[1])
    rec = corpus.pack_record(apps=len(plan.shards[rank]), wall_ns=int(res.step_ms[0] * 1e6),
                             digest_sum=sum(res.digests.values()))
    recs = corpus.unpack_records(corpus.gather_records(rec))
    d, m = corpus.gather_digests(n, res.digests)
    cache = {str(i): {"app_digest": str(dig(i))} for i in range(n)}
    good = corpus.check_digests(d, m, cache)
    cache["3"]["app_digest"] = "1"                  # a wrong cached value must be reported
    bad = corpus.check_digests(d, m, cache)
    out.put((rank, corpus.combine(recs)["apps"], int(m.sum()), good["checked"], good["mismatches"],
             bad["mismatches"], shard.built))
    dist.destroy_process_group()


def test_rank_path_over_gloo_world2():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_rank_path_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in ps:
        p.start()
    res = sorted(q.get(timeout=180) for _ in range(2))
    for p in ps:
        p.join(timeout=60)
        assert p.exitcode == 0
    for rank, apps, built, checked, mism, bad, steps in res:
        assert apps == 40 and built == 40 and checked == 40
        assert mism == [] and bad == [3]
        assert steps == 2 + 3 + 1                       # warm-up, timed, counting step
