"""The device layout (layout.cu: node records, operand rows, fact offsets, field-row and
projection tables, edge records and V1-V6 computed by kernels over the uploaded descriptor
arrays) against the host layout (loader.cu, $GDROID_HOST_LAYOUT=1): every device
table byte for byte, the facts against the oracle, and the device's own validation verdicts."""
from __future__ import annotations

import copy

import numpy as np
import pytest

import oracle
import paper_conf_ipps_yuwobby20_b200 as gd
from paper_conf_ipps_yuwobby20_b200._binding import GdroidError
from programs import tiny, tiny2, tiny_args
from synth import random_tiny
from synth import generator as G

pytestmark = pytest.mark.gpu

TABLES = ["nodes", "edges", "inl", "frow", "xmap", "args", "row_ptr", "arg_ptr", "node_method"]


def _tables(gs, monkeypatch, host):
    if host:
        monkeypatch.setenv("GDROID_HOST_LAYOUT", "1")
    else:
        monkeypatch.delenv("GDROID_HOST_LAYOUT", raising=False)
    app = gd.load(gs)
    t = [app.table(i) for i in range(len(TABLES))]
    return app, t


def _same_layout(gs, monkeypatch):
    a_dev, t_dev = _tables(gs, monkeypatch, host=False)
    a_host, t_host = _tables(gs, monkeypatch, host=True)
    monkeypatch.delenv("GDROID_HOST_LAYOUT", raising=False)
    for name, x, y in zip(TABLES, t_dev, t_host):
        assert x.size == y.size, f"{name}: {x.size} vs {y.size} bytes"
        if not np.array_equal(x, y):
            w = 64 if name == "nodes" else 32 if name == "edges" else 16 if name == "inl" else 4
            bad = np.nonzero((x != y).reshape(-1, w).any(axis=1))[0]
            raise AssertionError(f"{name}: {bad.size} records differ, first {bad[:8].tolist()}")
    a_host.free()
    return a_dev


@pytest.mark.parametrize("chunk", range(2))
def test_layout_random_tiny_batch(chunk, monkeypatch):
    """150 random tiny ICFGs (narrow and wide pools, arity up to 5, recursion) in one batch:
    identical tables, then facts = oracle."""
    gs = [random_tiny(s) for s in range(chunk * 150, chunk * 150 + 150)]
    app = _same_layout(gs, monkeypatch)
    app.build()
    digs = app.app_digests()
    for k, g in enumerate(gs):
        assert int(digs[k]) == oracle.build_idfg(g).app_digest, g.name


def test_layout_goldens(monkeypatch):
    gs = [tiny()[0], tiny(m2_entry=True)[0], tiny2()[0], tiny_args()[0], tiny_args(wide_pad=100)[0]]
    app = _same_layout(gs, monkeypatch)
    app.build()
    for k, g in enumerate(gs):
        r = oracle.build_idfg(g)
        ptr, pairs = app.read_all_facts(k)
        assert np.array_equal(ptr, r.ptr) and np.array_equal(pairs, r.pairs), g.name


@pytest.mark.parametrize("which", ["corpus", "worst"])
def test_layout_full_size(which, monkeypatch):
    """Corpus apps in one batch (dense (module, field) / (module, module) tables of several
    apps, one app > 820K nodes) and the worst preset (|Q| = 256 wide blocks)."""
    gs = [G.corpus_app(i) for i in (0, 1, 2, 729)] if which == "corpus" else [G.preset("worst")]
    app = _same_layout(gs, monkeypatch)
    app.free()


def _mut(g, **kw):
    h = copy.deepcopy(g)
    for k, v in kw.items():
        setattr(h, k, v)
    return h


def _invalid_cases():
    g = tiny()[0]
    out = []
    mp = g.method_n_params.copy(); mp[1] = 2
    ml = g.method_n_locals.copy(); ml[1] = 4
    out.append(("arity V6", _mut(g, method_n_params=mp, method_n_locals=ml), -1))
    ops = g.node_ops.copy(); ops[9, 1] = 6
    out.append(("operand local of another method V4", _mut(g, node_ops=ops), -2))
    ek = g.edge_kind.copy(); col = g.col.copy()
    e = int(np.nonzero(ek == 2)[0][0]); col[e] = 7
    out.append(("RET edge to a non-RETSITE V5", _mut(g, col=col), -1))
    col = g.col.copy(); col[0] = g.n_nodes + 5
    out.append(("edge target out of range", _mut(g, col=col), -1))
    ek = g.edge_kind.copy(); ek[0] = 7
    out.append(("bad edge kind", _mut(g, edge_kind=ek), -1))
    nk = g.node_kind.copy(); nk[int(np.nonzero(g.node_kind == 0)[0][0])] = 16
    out.append(("bad node kind", _mut(g, node_kind=nk), -1))
    ops = g.node_ops.copy()
    n_new = int(np.nonzero(g.node_kind == 7)[0][0]); ops[n_new, 3] = 0
    out.append(("NEW of NULL", _mut(g, node_ops=ops), -1))
    ops = g.node_ops.copy()
    n_ld = int(np.nonzero(g.node_kind == 12)[0][0]); ops[n_ld, 2] = 99
    out.append(("field out of range", _mut(g, node_ops=ops), -1))
    rp = g.row_ptr.copy()
    i = int([j for j in range(1, g.n_nodes - 1) if rp[j + 1] > rp[j]][0])
    rp[i] = rp[i + 1] + 1                        # node i: row_ptr[i] > row_ptr[i + 1]
    out.append(("row_ptr not monotone", _mut(g, row_ptr=rp), -1))
    # a C2R edge whose target RETSITE names another CALL
    ops = g.node_ops.copy(); n_rs = int(np.nonzero(g.node_kind == 3)[0][0]); ops[n_rs, 3] = 0
    out.append(("RETSITE without its CALL", _mut(g, node_ops=ops), -1))
    return out


@pytest.mark.parametrize("device_only", [False, True])
def test_layout_rejects_invalid(device_only, monkeypatch):
    """Every invalid input is rejected by the layout kernels (GDROID_DL_DEVICE_ERRORS=1: their own
    status) and, by default, with the host validator's exact status and message."""
    if device_only:
        monkeypatch.setenv("GDROID_DL_DEVICE_ERRORS", "1")
    for name, h, want in _invalid_cases():
        with pytest.raises(GdroidError) as e:
            gd.load([random_tiny(3), h])             # the invalid app is app 1 of a batch
        assert e.value.code == want, f"{name}: {e.value}"
        if device_only:
            assert "device layout" in str(e.value) and "app 1" in str(e.value), name
        monkeypatch.setenv("GDROID_HOST_LAYOUT", "1")
        with pytest.raises(GdroidError) as e2:
            gd.load([random_tiny(3), h])
        monkeypatch.delenv("GDROID_HOST_LAYOUT")
        assert e2.value.code == want, name
        if not device_only:
            assert str(e.value) == str(e2.value), name
