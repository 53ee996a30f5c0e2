#!/usr/bin/env python3
"""bench.py — IDFG construction throughput on B200 (one process per GPU).

Metric (BASELINE.json): "IDFG build ms/app and node-visits/s (1 GPU); corpus apps/s at
1/2/4/8 B200".  A *step* is one pass of the whole hot path (zero the
fact store, seed, fixed point, digests) over one batch of synthetic apps resident in HBM.

Workloads (--workload):
  corpus  (default) each rank builds a fixed shard of B apps of the seeded 1000-app corpus
          (BASELINE.json configs[4]; apps 0..B*N-1, LPT-sharded by estimated size) as ONE
          batch handle: weak scaling (per-rank app count fixed as N grows).
  median / small / worst   one app of that preset per rank (replicas).
value = apps built by all ranks / max-over-ranks device time of the K timed steps.

--impl reference runs the CPU oracle (oracle/, the reference arm of this tier) on a bounded
sample of the same workload on the host cores; rank 0 only.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "IDFG build ms/app and node-visits/s (1 GPU); corpus apps/s at 1/2/4/8 B200"


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--workload", default="corpus", choices=["corpus", "median", "small", "worst"])
    ap.add_argument("--apps-per-rank", type=int, default=8)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--loop-mode", type=int, default=0)
    ap.add_argument("--variant", default="default", choices=["default", "mat", "mat_grp", "gdroid", "plain"],
                    help="ablation variant (SURVEY §8(f) 1); plain needs one app per rank")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-seconds", type=float, default=12.0)
    ap.add_argument("--e2e-steps", type=int, default=5)
    return ap.parse_args()


# ------------------------------------------------------------------ workload construction
def workload_apps(args, rank, world):
    """Returns (list of Icfg for this rank, description dict).  Generation is not timed."""
    from synth import generator as G
    if args.workload != "corpus":
        g = G.preset(args.workload)
        return [g], {"workload": f"{args.workload} app (seed {G.PRESETS[args.workload].seed})",
                     "apps_per_rank": 1}
    B = args.apps_per_rank
    n_total = B * world
    sizes = G.corpus_sizes(n_total)
    order = sorted(range(n_total), key=lambda i: -sizes[i])       # LPT by estimated cost
    loads = [0] * world
    shard = [[] for _ in range(world)]
    for i in order:
        r = min(range(world), key=lambda q: (loads[q], q) if len(shard[q]) < B else (1 << 62, q))
        shard[r].append(i)
        loads[r] += sizes[i]
    mine = sorted(shard[rank])
    apps = [G.corpus_app(i) for i in mine]
    return apps, {"workload": f"corpus shard: apps {n_total} of the seeded 1000-app corpus "
                              f"(seeds 1000..{1000 + n_total - 1}), {B} per rank",
                  "apps_per_rank": B, "app_ids": mine}


# ------------------------------------------------------------------ clocks sampling
class Clocks:
    def __init__(self, device):
        self.samples = []
        self.device = device
        self.proc = None

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", f"--id={self.device}",
                 "--query-gpu=clocks.sm,clocks.max.sm,utilization.gpu,clocks_event_reasons.active,"
                 "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
                 "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap",
                 "--format=csv,noheader,nounits", "-lms", "100"],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None
        return self

    def _read(self):
        for line in self.proc.stdout:
            self.samples.append([x.strip() for x in line.split(",")])

    def __exit__(self, *a):
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=2)
            except Exception:
                self.proc.kill()

    def summary(self):
        if not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unsampled"], "samples": 0}
        sm = [int(s[0]) for s in self.samples if s[0].isdigit()]
        mx = [int(s[1]) for s in self.samples if s[1].isdigit()]
        busy = [int(s[0]) for s in self.samples if s[0].isdigit() and s[2].isdigit() and int(s[2]) > 0]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = set()
        for s in self.samples:
            for k, nm in enumerate(names):
                if len(s) > 4 + k and s[4 + k].lower().startswith("active"):
                    reasons.add(nm)
        return {"sm_mhz": statistics.median(busy or sm) if sm else None,
                "sm_max_mhz": max(mx) if mx else None, "reasons": sorted(reasons),
                "samples": len(self.samples), "samples_busy": len(busy)}


def measured_peak():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        with open(p) as fh:
            return float(json.load(fh)["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    except Exception:
        return 6650.0, "fallback (B200_PROFILING.md: 6.65 TB/s)"


def ncu_traffic(workload, apps_per_rank):
    """Per-launch DRAM bytes of k_fixpoint from the committed ncu summary of THIS workload
    (profiles/ncu_summary.json, written by scripts/ncu_summary.py), else None."""
    p = os.path.join(ROOT, "profiles", "ncu_summary.json")
    try:
        with open(p) as fh:
            d = json.load(fh)
        for cap in d.get("captures", [d]):
            if cap.get("bench_workload") == workload and cap.get("apps_per_rank", apps_per_rank) == apps_per_rank:
                return cap.get("k_fixpoint", {}).get("dram_bytes_per_launch"), cap.get("workload")
    except Exception:
        pass
    return None, None


# ------------------------------------------------------------------ CPU oracle legs
def oracle_sample(apps, seconds):
    """Time the oracle (as it stands, single-threaded) on apps of the workload, cycling through
    them until about `seconds` of CPU work (at most 64 runs)."""
    import oracle
    t0 = time.perf_counter()
    done, visits, app_s = 0, 0, []
    while done < 64:
        g = apps[done % len(apps)]
        r = oracle.build_idfg(g)
        done += 1
        visits += r.visits
        app_s.append(r.seconds)
        if time.perf_counter() - t0 > seconds:
            break
    wall = time.perf_counter() - t0
    return {"apps": done, "wall_s": wall, "visits": visits, "oracle_s": sum(app_s),
            "digests": None}


def run_reference(args):
    """--impl reference: the oracle on host cores, same config/metric; rank 0 only."""
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    if rank != 0:
        return
    apps, desc = workload_apps(args, 0, 1)
    import oracle
    oracle.build()
    for i in range(args.warmup):
        oracle.build_idfg(apps[i % len(apps)])
    t0 = time.perf_counter()
    visits = 0
    for s in range(args.steps):                                  # one app per step (bounded)
        r = oracle.build_idfg(apps[s % len(apps)])
        visits += r.visits
    dt = time.perf_counter() - t0
    v = args.steps / dt
    line = {"impl": "reference", "metric": METRIC, "value": v, "unit": "apps/s",
            "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": dt / args.steps * 1e3, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "u64", "data": "synthetic (seeded generator)",
            "config": {**{k: v2 for k, v2 in desc.items() if k != "app_ids"},
                       "step": "oracle on one app of the workload (bounded sample)"},
            "node_visits_per_s": visits / dt,
            "cpu_baseline": {"value": v, "unit": "apps/s", "cores": 1, "kind": "oracle",
                             "sample": f"{args.steps} apps of the workload, single-threaded C++ oracle"},
            "e2e": {"value": v, "unit": "apps/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ------------------------------------------------------------------ the GPU arm
def run_ours(args):
    import numpy as np
    import torch
    import torch.distributed as dist

    import paper_conf_ipps_yuwobby20_b200 as gd

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    # ranks on one host share its cores: the library's loader pool gets an equal share
    per_host = int(os.environ.get("LOCAL_WORLD_SIZE", "1"))
    os.environ.setdefault("GDROID_HOST_THREADS", str(max(1, len(os.sched_getaffinity(0)) // max(1, per_host))))
    assert torch.cuda.is_available(), "bench needs a GPU"
    torch.cuda.set_device(local)
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    stream = torch.cuda.current_stream()
    apps, desc = workload_apps(args, rank, world)
    n_apps = len(apps)
    nodes = sum(g.n_nodes for g in apps)
    input_bytes = sum(g.nbytes() for g in apps)

    plain = args.variant == "plain"
    assert not plain or len(apps) == 1, "--variant plain takes one app per rank (--apps-per-rank 1)"
    app = gd.load(apps, device=local, stream=stream.cuda_stream, plain=plain)   # inputs resident in HBM
    for _ in range(args.warmup):
        app.build(loop_mode=args.loop_mode, variant=args.variant, byte_model=False)
    torch.cuda.synchronize()

    def barrier():
        if world > 1:
            dist.barrier()

    stats = []
    with Clocks(local) as clk:
        barrier()
        torch.cuda.synchronize()
        ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        ev0.record(stream)
        for _ in range(args.steps):
            stats.append(app.build(loop_mode=args.loop_mode, variant=args.variant, byte_model=False))
        ev1.record(stream)
        torch.cuda.synchronize()
        barrier()
    my_ms = ev0.elapsed_time(ev1)
    digests = app.app_digests()
    # the byte models are counted by one extra, untimed build of the same
    # workload with the counting instantiation of the kernel (same fixed point and schedule)
    counted = app.build(loop_mode=args.loop_mode, variant=args.variant, byte_model=True)
    assert np.array_equal(app.app_digests(), digests)

    # e2e: the public C-ABI calls with HOST buffers, every step: gdroid_load_batch (host tables +
    # pinned H2D), gdroid_build_idfg, gdroid_app_digests (D2H of the result).  Steps are
    # double-buffered like the paper's dual-buffering: a loader thread loads
    # step i+1 on its own stream while step i builds.
    import queue as _queue
    import threading as _threading
    e2e_ms, e2e_parts = [], []
    if args.e2e_steps > 0:
        streams = [torch.cuda.Stream(device=local), torch.cuda.Stream(device=local)]
        q = _queue.Queue(maxsize=1)
        load_ms = []

        def loader():
            for i in range(args.e2e_steps + 1):          # +1: the first load primes the pipeline
                t = time.perf_counter()
                a = gd.load(apps, device=local, stream=streams[i % 2].cuda_stream, plain=plain)
                load_ms.append((time.perf_counter() - t) * 1e3)
                q.put(a)

        th = _threading.Thread(target=loader, daemon=True)
        barrier()
        torch.cuda.synchronize()
        th.start()
        first = q.get()                                  # not timed: pipeline fill
        first.build(loop_mode=args.loop_mode, variant=args.variant, byte_model=False)
        assert np.array_equal(first.app_digests(), digests)
        first.free()
        t0 = time.perf_counter()
        for i in range(args.e2e_steps):
            tb = time.perf_counter()
            a2 = q.get()
            a2.build(loop_mode=args.loop_mode, variant=args.variant, byte_model=False)
            tc = time.perf_counter()
            d2 = a2.app_digests()                        # D2H of the result
            a2.free()
            assert np.array_equal(d2, digests)
            e2e_parts.append(((tc - tb) * 1e3,))
        e2e_total = (time.perf_counter() - t0) * 1e3
        th.join()
        e2e_ms = [e2e_total / args.e2e_steps]
        e2e_parts = [(statistics.median(load_ms[1:]), statistics.median(x[0] for x in e2e_parts), 0.0)]
    e2e_mine = statistics.median(e2e_ms) if e2e_ms else float("nan")

    fix_ns = [s["fixpoint_ns"] for s in stats]
    alg = counted["alg_bytes"]
    dense = counted["dense_bytes"]
    visits = stats[-1]["node_visits"]
    rec = torch.tensor([my_ms, e2e_mine, float(n_apps), float(visits), float(nodes),
                        float(statistics.mean(fix_ns)), float(alg)], dtype=torch.float64,
                       device="cuda")
    if world > 1:                                         # NCCL gather of per-rank records
        gathered = [torch.zeros_like(rec) for _ in range(world)]
        dist.all_gather(gathered, rec)
        dig = torch.tensor(digests.view(np.int64), device="cuda")
        dig_all = [torch.zeros_like(dig) for _ in range(world)]
        dist.all_gather(dig_all, dig)
        recs = torch.stack(gathered).cpu().numpy()
    else:
        recs = rec.unsqueeze(0).cpu().numpy()
    if rank != 0:
        if world > 1:
            dist.destroy_process_group()
        return

    max_ms = float(recs[:, 0].max())
    total_apps = float(recs[:, 2].sum())
    ms_step = max_ms / args.steps
    value = total_apps * args.steps / (max_ms / 1e3)
    e2e_max = float(recs[:, 1].max())
    fix_ms = statistics.mean(fix_ns) / 1e6
    peak, peak_src = measured_peak()
    achieved = alg / (statistics.mean(fix_ns) / 1e9) / 1e9     # GB/s, touched-word model
    traffic, traffic_wl = ncu_traffic(args.workload, desc["apps_per_rank"])
    clocks = clk.summary()
    line = {
        "metric": METRIC, "value": value, "unit": "apps/s", "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms_step,
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "u64",
        "data": "synthetic (seeded generator, Android-app-shaped ICFGs)",
        "config": {**{k: v for k, v in desc.items() if k != "app_ids"},
                   "nodes_per_rank": nodes, "input_bytes_per_rank": input_bytes,
                   "fact_store_bytes_per_rank": stats[-1]["fact_bytes"],
                   "l2": "fact store > L2 (126 MB) per step; re-zeroed each step",
                   "parallelism": f"apps sharded over {world} GPU(s), no data-path collective",
                   "loop_mode": args.loop_mode, "variant": args.variant},
        "ms_per_app": ms_step / (total_apps / world),
        "node_visits_per_s": float(recs[:, 3].sum()) * args.steps / (max_ms / 1e3),
        "rounds_per_step": stats[-1]["rounds"],
        "fixpoint_ms_per_step": fix_ms,
        "gpu_launches": int(stats[-1]["kernel_launches"]) * args.steps,
        "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                     "frac": achieved / peak, "traffic": traffic, "kernel": "k_fixpoint",
                     "bytes_model": "touched-word (SURVEY §8(d)); per launch = one step's fixed point (1-3 k_fixpoint launches under the hybrid light/heavy schedule, DESIGN.md §5.4; achieved = bytes / their summed CUDA-event time, traffic = ncu DRAM bytes summed over them); counted by one untimed build with the counting kernel instantiation, timed launches run without the counters",
                     "alg_bytes_per_launch": alg, "dense_bytes_per_launch": dense,
                     "dense_achieved": dense / (statistics.mean(fix_ns) / 1e9) / 1e9,
                     "peak_source": peak_src, "traffic_workload": traffic_wl},
        "e2e": {"value": total_apps / (e2e_max / 1e3), "unit": "apps/s",
                "h2d_bytes_per_step": input_bytes, "d2h_bytes_per_step": 8 * n_apps + 128,
                "ms_per_step": e2e_max,
                "pipeline": "double-buffered: load of step i+1 overlaps build of step i",
                "breakdown_ms": dict(zip(("load", "wait+build+readback"),
                                         [round(x, 2) for x in e2e_parts[0][:2]]))
                                if e2e_parts else None},
        "clocks": clocks,
    }
    if not args.no_cpu_baseline:
        import oracle
        oracle.build()
        s = oracle_sample(apps, args.cpu_seconds)
        line["cpu_baseline"] = {"value": s["apps"] / s["wall_s"], "unit": "apps/s", "cores": 1,
                                "kind": "oracle",
                                "sample": f"{s['apps']} oracle run(s) over rank 0's {len(apps)} app(s), "
                                          f"single-threaded ({s['wall_s']:.1f} s)",
                                "node_visits_per_s": s["visits"] / s["wall_s"]}
    print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()


def main():
    args = parse()
    if args.impl == "reference":
        run_reference(args)
    else:
        run_ours(args)


if __name__ == "__main__":
    main()
