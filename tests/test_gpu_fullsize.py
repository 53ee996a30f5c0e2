"""GPU parity at BASELINE.json's full sizes against stored oracle results.

tests/golden/oracle_digests.json is written by scripts/make_oracle_digests.py, which calls only
oracle/ (never the CUDA path).  At these sizes the comparison is: the app digest (C8), an
order-sensitive hash of the per-node digest array (so every node's set is checked), and the
complete pair lists of sampled nodes.  Corpus apps are built in batches (shared rounds), in
the same launch configuration bench.py times.
"""
from __future__ import annotations

import json
import os

import numpy as np
import pytest

import paper_conf_ipps_yuwobby20_b200 as gd
from synth import generator as G

pytestmark = pytest.mark.gpu
HERE = os.path.dirname(os.path.abspath(__file__))
FIX = os.path.join(HERE, "golden", "oracle_digests.json")
M = (1 << 64) - 1


def _mix64(z):
    z &= M
    z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & M
    z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & M
    return z ^ (z >> 31)


def _node_hash(per_node):
    """Order-sensitive hash of a per-node digest array (scripts/make_oracle_digests.py's
    node_hash), vectorised: uint64 arithmetic wraps mod 2^64 like the Python original."""
    d = np.asarray(per_node, dtype=np.uint64)
    with np.errstate(over="ignore"):
        z = (np.arange(len(d), dtype=np.uint64) * np.uint64(0x9E3779B97F4A7C15)) ^ d
        z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
        z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
        z = z ^ (z >> np.uint64(31))
        return int(z.sum(dtype=np.uint64))


def test_node_hash_matches_python_definition():
    rng = np.random.default_rng(5)
    per = rng.integers(0, 2**63, size=1000, dtype=np.uint64) * np.uint64(3)
    h = 0
    for i, d in enumerate(per.tolist()):
        h = (h + _mix64((i * 0x9E3779B97F4A7C15) ^ d)) & M
    assert _node_hash(per) == h


def _fixture():
    if not os.path.exists(FIX):
        pytest.skip("no stored oracle digests")
    return json.load(open(FIX))


def _check(app, k, g, ref):
    assert ref["gen_version"] == G.GEN_VERSION and ref["n_nodes"] == g.n_nodes
    for n, pairs in ref["samples"].items():
        got = app.read_facts(int(n), k=k)
        assert [str(int(p)) for p in got] == pairs, f"{ref['name']} node {n}"


@pytest.mark.parametrize("name,variant", [("small", "default"), ("median", "default"), ("worst", "default"),
                                          ("small", "mat"), ("median", "mat_grp"), ("median", "gdroid"),
                                          ("small", "plain"), ("small", "cell"), ("small", "sbda"),
                                          ("median", "sbda"), ("worst", "sbda")])
def test_preset_full_size(name, variant):
    fx = _fixture()
    if name not in fx:
        pytest.skip(f"{name} not in fixture")
    ref = fx[name]
    g = G.preset(name)
    app = gd.load(g, plain=(variant in ("plain", "cell")))
    app.build(variant=variant)
    per, dig = app.node_digests()
    assert str(dig) == ref["app_digest"]
    assert str(_node_hash(per)) == ref["node_digest_hash"]
    _check(app, 0, g, ref)


def test_corpus_batches_full_size():
    fx = _fixture()
    ids = [i for i in range(16) if f"corpus{i}" in fx]
    if not ids:
        pytest.skip("no corpus apps in fixture")
    for b0 in range(0, len(ids), 8):
        batch = ids[b0:b0 + 8]
        gs = [G.corpus_app(i) for i in batch]
        app = gd.load(gs)
        app.build()
        digs = app.app_digests()
        for k, (i, g) in enumerate(zip(batch, gs)):
            ref = fx[f"corpus{i}"]
            assert str(int(digs[k])) == ref["app_digest"], f"corpus{i}"
            _check(app, k, g, ref)
        app.free()


def test_corpus_run_shard_pipeline():
    """The corpus driver's per-rank pipeline (loader thread + batched builds) on 6 apps."""
    from paper_conf_ipps_yuwobby20_b200 import corpus
    fx = _fixture()
    ids = [i for i in range(6) if f"corpus{i}" in fx]
    sizes = G.corpus_sizes(16)
    res = corpus.run_shard(ids, G.corpus_app, sizes, node_budget=600_000)
    seen = {}
    for br in res:
        for k, i in enumerate(br.app_ids):
            seen[i] = str(int(br.digests[k]))
    assert sorted(seen) == ids and len(res) >= 2
    for i in ids:
        assert seen[i] == fx[f"corpus{i}"]["app_digest"]


# ---- the 1000-app corpus (BASELINE.json configs[4]) against tests/golden/corpus_digests.json
# (written by scripts/make_corpus_digests.py, which calls only oracle/), in the launch
# configuration bench.py times: corpus.plan_corpus batches (narrow apps under a 4M-node
# budget, each worst-shaped app alone) built by corpus.DeviceShard (tables resident, fact
# store released after every build).  Every app: app digest AND the order-sensitive hash of
# its per-node digest array (so every node's set is checked).
CFIX = os.path.join(HERE, "golden", "corpus_digests.json")


def _corpus_check(ids, node_budget=4_000_000):
    from paper_conf_ipps_yuwobby20_b200 import corpus
    if not os.path.exists(CFIX):
        pytest.skip("no stored corpus digests")
    fx = json.load(open(CFIX))
    assert fx["gen_version"] == G.GEN_VERSION
    ids = [i for i in ids if str(i) in fx["apps"]]
    assert ids
    n = max(ids) + 1
    sizes = G.corpus_sizes(n)
    wide = [G.corpus_config(i).q_cap > 64 for i in range(n)]
    plan = corpus.plan_corpus(sizes, wide, 1, node_budget=node_budget, app_ids=ids)
    checked = 0
    for b in plan.batches[0]:
        apps = corpus.make_apps(b, G.corpus_app, threads=min(16, len(os.sched_getaffinity(0))))
        sh = corpus.DeviceShard([b], apps)
        sh.step()
        sh.finish()
        h = sh.handles[0]
        digs = h.app_digests()
        for k, i in enumerate(b):
            ref = fx["apps"][str(i)]
            assert apps[i].n_nodes == ref["n_nodes"]
            assert str(int(digs[k])) == ref["app_digest"], f"corpus{i}"
            per, _ = h.node_digests(k)
            assert str(_node_hash(per)) == ref["node_digest_hash"], f"corpus{i} per-node"
            checked += 1
        sh.free()
    return checked


def test_corpus_digest_sample():
    """Every 20th app of the corpus (50 apps, 20K-2M nodes)."""
    assert _corpus_check(list(range(0, 1000, 20))) >= 45


def test_corpus_wide_apps():
    """The worst-shaped corpus apps (|Q| = 256) that the cache holds, each alone."""
    from synth import generator as G2
    wide = [i for i in range(1000) if G2.corpus_config(i).q_cap > 64]
    fx = json.load(open(CFIX)) if os.path.exists(CFIX) else {"apps": {}}
    have = [i for i in wide if str(i) in fx["apps"]]
    if not have:
        pytest.skip("no wide corpus apps in the cache yet")
    if os.environ.get("GDROID_QUICK"):
        have = have[:2]
    assert _corpus_check(have) == len(have)


@pytest.mark.skipif(bool(os.environ.get("GDROID_QUICK")), reason="GDROID_QUICK set (minutes on a B200)")
def test_corpus_digest_all():
    """All 1000 apps of the corpus that the cache holds (profiles/r02_full_corpus_parity.log)."""
    fx = json.load(open(CFIX)) if os.path.exists(CFIX) else {"apps": {}}
    assert _corpus_check(list(range(1000))) == len(fx["apps"]) >= 985
