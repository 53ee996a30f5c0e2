#!/usr/bin/env python3
"""Stall samples aggregated per CUDA source line (ncu --print-source cuda,sass)."""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
n = int(sys.argv[2]) if len(sys.argv) > 2 else 30
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
res = []
cur = None
for r in rows:
    if len(r) > 5 and r[0] not in ("", "Line No") and r[0].isdigit():
        try:
            res.append((float(r[4] or 0), int(r[0]), r[1].strip()[:90], r[7]))
        except ValueError:
            pass
tot = sum(x[0] for x in res)
print(f"total samples {tot:.0f}")
for s, ln, src, ex in sorted(res, reverse=True)[:n]:
    print(f"{100 * s / tot:6.2f}%  L{ln:<5d} {ex:>12s}  {src}")
