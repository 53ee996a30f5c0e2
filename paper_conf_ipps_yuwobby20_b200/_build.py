"""Compile libgdroid.so (the C-ABI library of include/gdroid.h) in-tree for sm_100a."""
from __future__ import annotations

import os
import subprocess

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
CSRC = os.path.join(HERE, "csrc")
LIB = os.path.join(HERE, "libgdroid.so")
SOURCES = [os.path.join(CSRC, f) for f in ("loader.cu", "kernels.cu", "plain.cu", "layout.cu")]
DEPS = SOURCES + [os.path.join(CSRC, "internal.cuh"), os.path.join(ROOT, "include", "gdroid.h")]
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
FLAGS = ["-gencode", "arch=compute_100a,code=sm_100a", "-lineinfo", "-O3", "-std=c++17",
         "-shared", "-Xcompiler", "-fPIC", "-Xptxas", "-v"]


FLAGS_FILE = LIB + ".flags"     # the extra nvcc flags the in-tree library was built with


def _built_flags():
    try:
        with open(FLAGS_FILE) as fh:
            return fh.read().strip()
    except OSError:
        return None


def build(force: bool = False, verbose: bool = False) -> str:
    """Rebuild when a source is newer than the library OR the library was built with other
    extra flags (GDROID_NVCC_FLAGS, used by A/B scripts) than the ones requested now, so an A/B
    variant left in the tree is never reused by a default build."""
    newest = max(os.path.getmtime(p) for p in DEPS)
    extra = os.environ.get("GDROID_NVCC_FLAGS", "").split()
    want = " ".join(extra)
    if (not force and os.path.exists(LIB) and os.path.getmtime(LIB) >= newest
            and _built_flags() == want):
        return LIB
    tmp = LIB + f".tmp{os.getpid()}"
    cmd = [NVCC, *FLAGS, *extra, "-I", os.path.join(ROOT, "include"), "-o", tmp, *SOURCES]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError("nvcc failed:\n" + r.stdout + r.stderr)
    if verbose:
        print(r.stderr)
    with open(os.path.join(HERE, "ptxas_info.txt"), "w") as fh:
        fh.write(r.stderr)
    os.replace(tmp, LIB)
    with open(FLAGS_FILE, "w") as fh:
        fh.write(want + "\n")
    return LIB


if __name__ == "__main__":
    print(build(force=True, verbose=True))
