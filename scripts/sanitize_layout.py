#!/usr/bin/env python3
"""compute-sanitizer workload for the device layout (layout.cu): valid batches (narrow and wide
pools, two corpus apps) and every invalid-input class of tests/test_gpu_layout.py, whose kernels
must reject the input without a single out-of-bounds access (GDROID_DL_DEVICE_ERRORS=1: the
kernels' own verdict, no host re-run)."""
import copy
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path[:0] = [ROOT, os.path.join(ROOT, "tests"), os.path.join(ROOT, "tests", "golden")]
os.environ["GDROID_DL_DEVICE_ERRORS"] = "1"
import paper_conf_ipps_yuwobby20_b200 as gd  # noqa: E402
from paper_conf_ipps_yuwobby20_b200._binding import GdroidError  # noqa: E402
from synth import generator as G  # noqa: E402
from synth import random_tiny  # noqa: E402
from test_gpu_layout import _invalid_cases  # noqa: E402

gs = [random_tiny(s, wide_pad=(100 if s % 3 == 0 else 0)) for s in range(64)] + [G.corpus_app(0), G.corpus_app(1)]
app = gd.load(gs)
app.build()
print("valid batch:", len(gs), "apps, digests", int(app.app_digests().sum()) & 0xffff)
app.free()
for name, h, want in _invalid_cases():
    try:
        gd.load([random_tiny(3), h])
        print("NOT REJECTED:", name)
        sys.exit(1)
    except GdroidError as e:
        assert e.code == want, (name, e.code, want)
        print("rejected:", name, e.code)
print("sanitize_layout ok")
