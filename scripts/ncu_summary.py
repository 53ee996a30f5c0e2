#!/usr/bin/env python3
"""Summarise an ncu report (--set full) and a launch-list CSV into profiles/ (text + JSON).

usage: ncu_summary.py REPORT.ncu-rep LAUNCHES.csv OUT_PREFIX [workload description]
"""
import csv
import io
import json
import subprocess
import sys
from collections import defaultdict

KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "lts__t_bytes.sum",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed", "launch__registers_per_thread",
        "launch__grid_size", "launch__block_size", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "smsp__inst_executed.sum", "smsp__sass_average_branch_targets_threads_uniform.pct",
        "l1tex__t_sector_hit_rate.pct", "lts__t_sector_hit_rate.pct"]


def kname(full):
    """'void gd::<unnamed>::k_fixpoint<(bool)1>(gd::Dev)' -> 'k_fixpoint'"""
    import re
    m = re.search(r"(k_[a-z_]+)", full)
    return m.group(1) if m else full.split("(")[0].split("::")[-1]


def raw(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units = rows[0], rows[1]
    res = []
    for r in rows[2:]:
        d = dict(zip(hdr, r))
        res.append((d, dict(zip(hdr, units))))
    return res


def stalls(d):
    tot = float(d.get("smsp__pcsamp_sample_count", "0").replace(",", "") or 0)
    out = {}
    for k, v in d.items():
        if k.startswith("smsp__pcsamp_warps_issue_stalled_") and not k.endswith("_not_issued"):
            try:
                x = float(v.replace(",", ""))
            except ValueError:
                continue
            if tot and x / tot > 0.005:
                out[k.replace("smsp__pcsamp_warps_issue_stalled_", "")] = round(100 * x / tot, 2)
    return dict(sorted(out.items(), key=lambda kv: -kv[1]))


def launches(path):
    per = defaultdict(list)
    with open(path) as fh:
        lines = [l for l in fh if l.startswith('"')]
    rd = csv.DictReader(io.StringIO("".join(lines)))
    for r in rd:
        if r.get("Metric Name") == "gpu__time_duration.sum":
            v = float(r["Metric Value"].replace(",", ""))
            unit = r.get("Metric Unit", "ns")
            scale = {"nsecond": 1e-6, "usecond": 1e-3, "msecond": 1.0, "ns": 1e-6, "us": 1e-3, "ms": 1.0}.get(unit, 1e-6)
            name = kname(r["Kernel Name"])
            per[name].append(v * scale)
    tot = sum(sum(v) for v in per.values())
    return {k: {"launches": len(v), "total_ms": round(sum(v), 4), "share": round(sum(v) / tot, 4)}
            for k, v in sorted(per.items(), key=lambda kv: -sum(kv[1]))}


def main():
    rep, lcsv, prefix = sys.argv[1:4]
    wl = sys.argv[4] if len(sys.argv) > 4 else ""
    summary = {"workload": wl, "launch_list": launches(lcsv) if lcsv != "-" else None}
    if len(sys.argv) > 5:
        summary["bench_workload"] = sys.argv[5]
        summary["apps_per_rank"] = int(sys.argv[6]) if len(sys.argv) > 6 else 1
    # Several captured launches of one kernel (the hybrid schedule runs k_fixpoint 1-3 times per
    # build) are summed: dram_bytes_per_launch = bytes of one build (all its
    # launches); the other metrics are those of the longest launch.
    tscale = {"nsecond": 1e-6, "usecond": 1e-3, "msecond": 1.0}
    for d, u in raw(rep):
        name = kname(d.get("Kernel Name", "?"))
        m = {k: d.get(k) for k in KEYS if k in d}
        m["units"] = {k: u.get(k) for k in KEYS if k in d}
        m["stall_pct"] = stalls(d)
        rd = float(d.get("dram__bytes_read.sum", "0").replace(",", "") or 0)
        wr = float(d.get("dram__bytes_write.sum", "0").replace(",", "") or 0)
        scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}
        m["dram_bytes_per_launch"] = rd * scale.get(u.get("dram__bytes_read.sum"), 1) + \
            wr * scale.get(u.get("dram__bytes_write.sum"), 1)
        ms = float(d.get("gpu__time_duration.sum", "0").replace(",", "") or 0) * \
            tscale.get(u.get("gpu__time_duration.sum"), 1.0)
        if name in summary:
            prev = summary[name]
            m["launches_captured"] = prev["launches_captured"] + 1
            m["total_ms_captured"] = prev["total_ms_captured"] + ms
            m["dram_bytes_per_launch"] += prev["dram_bytes_per_launch"]
            if prev["_ms"] > ms:
                keep = {k: m[k] for k in ("launches_captured", "total_ms_captured", "dram_bytes_per_launch")}
                m = dict(prev, **keep)
                ms = prev["_ms"]
        else:
            m["launches_captured"] = 1
            m["total_ms_captured"] = ms
        m["_ms"] = ms
        summary[name] = m
    for m in summary.values():
        if isinstance(m, dict):
            m.pop("_ms", None)
    with open(prefix + ".json", "w") as fh:
        json.dump(summary, fh, indent=1)
    print(json.dumps(summary, indent=1))


if __name__ == "__main__":
    main()
