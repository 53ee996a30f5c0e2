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
