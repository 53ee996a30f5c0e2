#!/usr/bin/env python3
"""Warp instructions executed per CUDA source line (ncu --page source, cuda+sass), sorted."""
import csv, io, subprocess, sys
from collections import defaultdict
rep = sys.argv[1]; n = int(sys.argv[2]) if len(sys.argv) > 2 else 40
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
agg = defaultdict(float); src = {}; fname = ""
for r in csv.reader(io.StringIO(out)):
    if len(r) == 2 and r[0] == "File Path":
        fname = r[1].split("/")[-1]
    if len(r) > 8 and r[0].isdigit() and r[2] == "-":
        try:
            agg[(fname, int(r[0]))] += float(r[7] or 0); src[(fname, int(r[0]))] = r[1].strip()[:95]
        except ValueError:
            pass
tot = sum(agg.values())
print(f"total warp instructions {tot:.3e}")
for k, v in sorted(agg.items(), key=lambda kv: -kv[1])[:n]:
    print(f"{100 * v / tot:6.2f}%  {k[0]}:{k[1]:<5d} {src[k]}")
