"""The seeded input generators cover what the CALL edge transform (SURVEY §8(c) C3,
PAPER.md:758-766) must handle: calls with more than 3 parameters (the args-table path of the
CUDA loader/kernels) and one local passed as 4 or more actuals (one source row feeding many
parameter rows), in narrow and wide pools.  Input construction only; no oracle call."""
from __future__ import annotations

import numpy as np

from synth import generator as G
from synth import random_tiny
from synth.icfg import CALL
from synth.reductions import random_inline_pair


def _arity_stats(gs):
    max_ar, max_rep = 0, 0
    for g in gs:
        ap = g.call_arg_ptr.astype(np.int64)
        for n in np.nonzero(g.node_kind == CALL)[0]:
            a = g.call_args[ap[n]:ap[n + 1]]
            max_ar = max(max_ar, len(a))
            pos = a[a >= 0]
            if len(pos):
                max_rep = max(max_rep, int(np.bincount(pos).max()))
    return max_ar, max_rep


def test_tiny_random_arity_and_repeats():
    # the seeds of tests/test_gpu_parity.py's narrow and wide batches
    narrow = [random_tiny(s) for s in range(0, 150)]
    wide = [random_tiny(s, wide_pad=150) for s in range(5150, 5270)]
    for gs in (narrow, wide):
        ar, rep = _arity_stats(gs)
        assert ar >= 5 and rep >= 4, (ar, rep)


def test_inline_pairs_arity():
    gs = [random_inline_pair(s)[0] for s in range(300)]
    ar, rep = _arity_stats(gs)
    assert ar >= 6 and rep >= 4, (ar, rep)


def test_app_generator_arity_0_to_8():
    g = G.preset("small")
    ap = np.diff(g.call_arg_ptr.astype(np.int64))
    hist = np.bincount(ap[g.node_kind == CALL], minlength=9)
    assert hist[4:].sum() > 0 and hist[8] > 0, hist
    ar, rep = _arity_stats([g])
    assert ar == 8 and rep >= 4, (ar, rep)
    assert G.GEN_VERSION >= 2
