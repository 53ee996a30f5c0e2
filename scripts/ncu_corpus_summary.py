#!/usr/bin/env python3
"""Summarise an ncu launch CSV of `bench.py --steps 1 --warmup 0` (metrics dram__bytes_read.sum,
dram__bytes_write.sum, gpu__time_duration.sum) into the corpus1000 capture of
profiles/ncu_summary.json: per-kernel time shares of the timed step and the DRAM bytes of its
k_fixpoint launches (the counting step's instantiations, CNT = 1, are excluded).
usage: ncu_corpus_summary.py LAUNCHES.csv [description]"""
import collections, csv, io, json, os, re, sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
path = sys.argv[1]
desc = sys.argv[2] if len(sys.argv) > 2 else "corpus1000, bench.py --steps 1 --warmup 0"
lines = [l for l in open(path) if l.startswith('"')]
per = collections.defaultdict(dict)
for r in csv.DictReader(io.StringIO("".join(lines))):
    per[(int(r["ID"]), r["Kernel Name"])][r["Metric Name"]] = float(r["Metric Value"].replace(",", ""))
shares, nl, fix = collections.defaultdict(float), collections.Counter(), [0, 0.0, 0.0]
for (i, k), d in sorted(per.items()):
    m = re.search(r"(k_[a-z_]+)(<([^>]*)>)?", k)
    nm, targs = m.group(1), m.group(3)
    if nm in ("k_fixpoint", "k_sbda") and targs and targs.split(",")[1].strip() == "1":
        continue                                            # the counting step
    ms = d.get("gpu__time_duration.sum", 0) / 1e6
    shares[nm] += ms
    nl[nm] += 1
    if nm == "k_fixpoint":
        fix[0] += 1; fix[1] += ms
        fix[2] += d.get("dram__bytes_read.sum", 0) + d.get("dram__bytes_write.sum", 0)
for k in ("k_digest", "k_seed"):                            # these ran in both builds of the run
    shares[k] /= 2; nl[k] //= 2
tot = sum(shares.values())
out = {"bench_workload": "corpus1000", "workload": desc,
       "launch_list": {k: {"launches": nl[k], "total_ms": round(v, 3), "share": round(v / tot, 4)}
                       for k, v in sorted(shares.items(), key=lambda kv: -kv[1])},
       "k_fixpoint": {"launches_captured": fix[0], "total_ms_captured": round(fix[1], 3),
                      "dram_bytes_per_launch": fix[2],
                      "note": "DRAM bytes of all k_fixpoint launches of one step (timed instantiations), "
                              "summed like alg_bytes_per_launch"}}
p = os.path.join(ROOT, "profiles", "ncu_summary.json")
d = json.load(open(p))
caps = [c for c in d.get("captures", [d]) if c.get("bench_workload") != "corpus1000"] + [out]
json.dump({"captures": caps}, open(p, "w"), indent=1)
print(json.dumps(out, indent=1))
