#!/usr/bin/env python3
"""Top SASS instructions by stall samples (with their stall-reason columns) of an ncu report."""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
n = int(sys.argv[2]) if len(sys.argv) > 2 else 30
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hdr = rows[1]
data = rows[2:]
i_s = hdr.index("Warp Stall Sampling (All Samples)")
i_src = hdr.index("Source")
i_ex = hdr.index("Instructions Executed")
tot = sum(float(r[i_s] or 0) for r in data)
print(f"total samples {tot:.0f}")
for idx, r in sorted(enumerate(data), key=lambda t: -float(t[1][i_s] or 0))[:n]:
    print(f"{100 * float(r[i_s]) / tot:6.2f}% {r[i_ex]:>12s} [{idx:5d}] {r[i_src][:100]}")
