#!/usr/bin/env python3
"""bench.py — IDFG construction throughput on B200 (one process per GPU).

Metric (BASELINE.json): "IDFG build ms/app and node-visits/s (1 GPU); corpus apps/s at
1/2/4/8 B200".  A *step* is one pass of the whole hot path (zero the
fact store, seed, fixed point, digests) over the workload, inputs resident in HBM.

Workloads (--workload):
  corpus1000 (default) the seeded 1000-app corpus of BASELINE.json configs[4] (LogNormal
          sizes, 20K-2M nodes, the clipped 1.5 % tail in the worst-case |Q| = 256 shape),
          LPT-sharded over the ranks by estimated cost: STRONG scaling (the corpus is fixed,
          N ranks split it).  Every rank keeps all its batches' tables in HBM; a batch holds a
          fact store only while it builds.  value = 1000 apps / max-over-ranks
          device time per step.  Rank 0 also builds the small / median / worst presets alone
          (the metric's "IDFG build ms/app and node-visits/s (1 GPU)", `per_config`).
  corpus8  the round-1 workload: 8 apps per rank as one batch (weak scaling).
  small / median / worst   one app of that preset per rank (replicas).

--impl reference runs the CPU oracle (oracle/, the reference arm of this tier) on a bounded
sample of the same workload on the host cores (rank 0 only).
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

# single-thread oracle throughput on narrow corpus apps (~10.6 us per node, tests/golden/
# corpus_digests.json oracle_s): sizes the bounded CPU samples
ORACLE_NODES_PER_CORE_S = 9.0e4
METRIC = "IDFG build ms/app and node-visits/s (1 GPU); corpus apps/s at 1/2/4/8 B200"
CORPUS_CACHE = os.path.join(ROOT, "tests", "golden", "corpus_digests.json")
PRESET_CACHE = os.path.join(ROOT, "tests", "golden", "oracle_digests.json")


def parse(argv=None):
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=3)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--workload", default="corpus1000",
                    choices=["corpus1000", "corpus8", "median", "small", "worst"])
    ap.add_argument("--n-apps", type=int, default=1000, help="corpus1000: apps of the corpus")
    ap.add_argument("--apps-per-rank", type=int, default=8, help="corpus8: apps per rank")
    ap.add_argument("--node-budget", type=int, default=16_000_000, help="narrow apps per batch (nodes)")
    ap.add_argument("--wide-per-batch", type=int, default=1)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-per-config", action="store_true")
    ap.add_argument("--cpu-seconds", type=float, default=15.0)
    ap.add_argument("--e2e-steps", type=int, default=1)
    ap.add_argument("--e2e-readback", default="facts", choices=["facts", "digests"])
    ap.add_argument("--e2e-reserve-sms", type=int, default=0,
                    help="SMs the e2e builds leave free for the previous batch's readback kernels")
    ap.add_argument("--gen-threads", type=int, default=0)
    return ap.parse_args(argv)


def host_threads():
    return len(os.sched_getaffinity(0))


def cpu_model():
    try:
        out = subprocess.run(["lscpu"], capture_output=True, text=True).stdout
        for line in out.splitlines():
            if line.startswith("Model name"):
                return line.split(":", 1)[1].strip()
    except Exception:
        pass
    return "unknown"


# ------------------------------------------------------------------ workload construction
def workload(args, world):
    """(plan, make_app, desc).  Generation is never timed."""
    from paper_conf_ipps_yuwobby20_b200 import corpus
    from synth import generator as G
    if args.workload == "corpus1000":
        n = args.n_apps
        cfgs = [G.corpus_config(i) for i in range(n)]
        sizes = G.corpus_sizes(n)
        wide = [c.q_cap > 64 for c in cfgs]
        plan = corpus.plan_corpus(sizes, wide, world, node_budget=args.node_budget,
                                  wide_per_batch=args.wide_per_batch)
        desc = {"workload": f"corpus{n}: the seeded {n}-app corpus (BASELINE.json configs[4]; seeds "
                            f"1000..{999 + n}; {sum(wide)} worst-shaped apps), LPT-sharded over "
                            f"{world} rank(s), strong scaling",
                "n_apps": n, "node_budget": args.node_budget, "wide_per_batch": args.wide_per_batch}
        return plan, G.corpus_app, desc, "strong"
    if args.workload == "corpus8":
        B = args.apps_per_rank
        n = B * world
        sizes = G.corpus_sizes(n)
        wide = [G.corpus_config(i).q_cap > 64 for i in range(n)]
        plan = corpus.plan_corpus(sizes, wide, world, node_budget=1 << 62, per_rank=B)
        plan.batches = [[sorted(s)] for s in plan.shards]          # one batch per rank
        desc = {"workload": f"corpus shard: {B} apps per rank of the seeded corpus (seeds 1000..{999 + n}), "
                            f"one batch per rank, weak scaling", "apps_per_rank": B}
        return plan, G.corpus_app, desc, "weak"
    # presets: one app per rank (replicas), app id = rank
    cfg = G.PRESETS[args.workload]
    plan = corpus.Plan(world, world, [0] * world, [cfg.q_cap > 64] * world,
                       [[r] for r in range(world)], [[[r]] for r in range(world)])
    desc = {"workload": f"{args.workload} app (seed {cfg.seed}), one per rank (replicas)"}
    return plan, (lambda i: G.preset(args.workload)), desc, "weak"


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


def ncu_traffic(workload):
    """DRAM bytes of k_fixpoint per step of THIS workload from the committed ncu summary
    (profiles/ncu_summary.json, written by scripts/ncu_summary.py), else (None, None)."""
    p = os.path.join(ROOT, "profiles", "ncu_summary.json")
    try:
        with open(p) as fh:
            d = json.load(fh)
        for cap in d.get("captures", [d]):
            if cap.get("bench_workload") == workload:
                return cap.get("k_fixpoint", {}).get("dram_bytes_per_launch"), cap.get("workload")
    except Exception:
        pass
    return None, None


# ------------------------------------------------------------------ CPU oracle legs
def oracle_sample_ids(plan, budget_nodes):
    """A size-stratified sample of the workload's narrow apps (evenly spaced in size order)
    whose node count is about budget_nodes.  Worst-shaped apps (~800 s of one core each) are
    excluded from the timed sample and reported separately."""
    ids = sorted((i for s in plan.shards for i in s if not plan.wide[i]), key=lambda i: plan.sizes[i])
    if not ids:
        return []
    tot = sum(plan.sizes[i] for i in ids)
    k = max(1, min(len(ids), round(len(ids) * budget_nodes / max(tot, 1))))
    step = len(ids) / k
    return sorted({ids[int(j * step + step / 2)] for j in range(k)})


def oracle_pool(apps, threads):
    """Run the oracle (as it stands, single-threaded code) on every app with `threads`
    concurrent workers; returns (wall s, Σ oracle s, Σ visits, digests)."""
    from concurrent.futures import ThreadPoolExecutor
    import oracle
    t0 = time.perf_counter()
    with ThreadPoolExecutor(max_workers=threads) as ex:
        res = list(ex.map(oracle.run_timed, apps))
    wall = time.perf_counter() - t0
    return wall, sum(r[0] for r in res), sum(r[1] for r in res), [r[2] for r in res]


def run_reference(args):
    """--impl reference: the oracle on the host cores, same workload/metric; rank 0 only.
    Each step = one bounded, size-stratified sample of the workload's apps run by P threads."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    import oracle
    oracle.build()
    plan, make_app, desc, scaling = workload(args, 1)
    P = host_threads()
    per_step_nodes = ORACLE_NODES_PER_CORE_S * P * 4.0   # ~4 s of P threads per step
    ids = oracle_sample_ids(plan, per_step_nodes * (args.steps + args.warmup))
    if not ids:                                          # a preset workload: its one app
        ids = plan.shards[0]
    apps = [make_app(i) for i in ids]
    nsteps = args.steps + args.warmup
    chunks = [apps[j::nsteps] for j in range(nsteps)] if len(apps) >= nsteps else [apps] * nsteps
    for j in range(args.warmup):
        oracle_pool(chunks[j], P)
    wall, n_apps, visits, nodes = 0.0, 0, 0, 0
    for j in range(args.warmup, nsteps):
        w, _, v, _ = oracle_pool(chunks[j], P)
        wall += w
        n_apps += len(chunks[j])
        visits += v
        nodes += sum(a.n_nodes for a in chunks[j])
    v = n_apps / wall
    sample = (f"{n_apps} apps in {args.steps} steps (size-stratified sample of the workload's "
              f"narrow apps, {nodes} nodes), oracle on {P} host threads")
    line = {"impl": "reference", "metric": METRIC, "value": v, "unit": "apps/s",
            "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": wall / args.steps * 1e3, "higher_is_better": True, "scaling": scaling,
            "vs_baseline": None, "dtype": "u64", "data": "synthetic (seeded generator)",
            "config": {**desc, "step": "oracle on a bounded sample of the workload"},
            "node_visits_per_s": visits / wall,
            "cpu_baseline": {"value": v, "unit": "apps/s", "cores": P, "kind": "oracle",
                             "sample": sample, "cpu_model": cpu_model()},
            "e2e": {"value": v, "unit": "apps/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ------------------------------------------------------------------ the GPU arm
def per_config_runs(device, stream, reps=5):
    """The metric's single-GPU figures: each preset built alone (1 warm-up, `reps` timed
    builds, CUDA events of the build; median), checked against the stored oracle digests."""
    import paper_conf_ipps_yuwobby20_b200 as gd
    from synth import generator as G
    cache = json.load(open(PRESET_CACHE)) if os.path.exists(PRESET_CACHE) else {}
    out = {}
    for name in ("small", "median", "worst"):
        g = G.preset(name)
        app = gd.load(g, device=device, stream=stream)
        app.build(byte_model=False)
        st = [app.build(byte_model=False) for _ in range(reps)]
        cnt = app.build(byte_model=True)
        dig = int(app.app_digests()[0])
        ref = cache.get(name, {})
        ms = statistics.median(s["build_ns"] for s in st) / 1e6
        fix_ms = statistics.median(s["fixpoint_ns"] for s in st) / 1e6
        out[name] = {"nodes": g.n_nodes, "ms_per_app": ms, "fixpoint_ms": fix_ms,
                     "node_visits_per_s": st[-1]["node_visits"] / (ms / 1e3),
                     "rounds": st[-1]["rounds"], "us_per_round": 1e3 * fix_ms / max(1, st[-1]["rounds"]),
                     "alg_gbs": cnt["alg_bytes"] / (fix_ms / 1e3) / 1e9,
                     "parity": ("ok" if str(dig) == ref.get("app_digest") else
                                ("MISMATCH" if ref else "no oracle cache"))}
        app.free()
    return out


def run_ours(args):
    import numpy as np
    import torch
    import torch.distributed as dist

    from paper_conf_ipps_yuwobby20_b200 import corpus

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    per_host = int(os.environ.get("LOCAL_WORLD_SIZE", "1"))
    nthreads = max(1, host_threads() // max(1, per_host))
    os.environ.setdefault("GDROID_HOST_THREADS", str(nthreads))
    assert torch.cuda.is_available(), "bench needs a GPU"
    # GDROID_BENCH_SHARE_GPU=1 (test hook): every rank on cuda:0 with gloo collectives, to run the
    # multi-rank path on a one-GPU box; the driver's runs use one GPU per rank and NCCL
    share = os.environ.get("GDROID_BENCH_SHARE_GPU") == "1"
    if share:
        local = 0
    torch.cuda.set_device(local)
    if world > 1:
        if share:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    dev = torch.device("cuda", local)
    cdev = None if share else dev                         # where collective tensors live
    stream = torch.cuda.current_stream()

    def barrier():
        if world > 1:
            dist.barrier()

    plan, make_app, desc, scaling = workload(args, world)
    my_batches = plan.batches[rank]
    my_ids = [i for b in my_batches for i in b]
    apps = corpus.make_apps(my_ids, make_app, threads=args.gen_threads or nthreads)
    shard = corpus.DeviceShard(my_batches, apps, device=local, stream=stream.cuda_stream)
    nodes = sum(shard.nodes)
    torch.cuda.synchronize()

    def timer(fn):
        ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        ev0.record(stream)
        fn()
        ev1.record(stream)
        torch.cuda.synchronize()
        return ev0.elapsed_time(ev1)

    with Clocks(local) as clk:
        res = corpus.run_rank(shard, args.steps, args.warmup, barrier, timer)
    clocks = clk.summary()
    stats, counted = res.stats, res.counted
    my_ms = res.step_ms[0]
    visits = sum(s["node_visits"] for s in stats)
    fix_ns = sum(s["fixpoint_ns"] for s in stats)
    alg = sum(s["alg_bytes"] for s in counted)
    dense = sum(s["dense_bytes"] for s in counted)
    launches = sum(s["kernel_launches"] for s in stats)
    batch_ms = [s["build_ns"] / 1e6 for s in stats]
    # per-app IDFG time: apps of a batch share its rounds; an app's share is its node fraction
    app_ms = []
    for b, s, nn in zip(my_batches, stats, shard.nodes):
        for i in b:
            app_ms.append(s["build_ns"] / 1e6 * apps[i].n_nodes / max(1, nn))
    rec = corpus.pack_record(apps=len(my_ids), visits=visits, alg_bytes=alg, build_ns=int(my_ms * 1e6),
                             wall_ns=int(my_ms * 1e6), max_app_ns=int(max(batch_ms) * 1e6),
                             digest_sum=sum(res.digests.values()), errors=0)
    recs = corpus.unpack_records(corpus.gather_records(rec, cdev if world > 1 else None))
    dig_all, dig_mask = corpus.gather_digests(plan.n_apps, res.digests, cdev if world > 1 else None)
    shard.free()

    # e2e through the public API from host arrays: load (host tables + pinned H2D) of batch i+1
    # overlapped with build + fact readback of batch i
    e2e = None
    if args.e2e_steps > 0:
        bufs = corpus.ReadbackBuffers()
        corpus.run_pipelined(my_batches, lambda i: apps[i], device=local, readback=args.e2e_readback,
                             bufs=bufs, reserve_sms=args.e2e_reserve_sms)   # untimed warm-up: sizes the pinned buffers
        barrier()
        torch.cuda.synchronize()
        d2h = h2d = 0
        t0 = time.perf_counter()
        for _ in range(args.e2e_steps):
            out = corpus.run_pipelined(my_batches, lambda i: apps[i], device=local, readback=args.e2e_readback,
                                       bufs=bufs, reserve_sms=args.e2e_reserve_sms)
            for br in out:
                for k, i in enumerate(br.app_ids):
                    if int(br.digests[k]) != res.digests[i]:
                        raise RuntimeError(f"e2e digest of app {i} differs from the device-resident run")
                d2h += br.d2h_bytes
                h2d += br.h2d_bytes
        torch.cuda.synchronize()
        e2e_ms = (time.perf_counter() - t0) * 1e3 / args.e2e_steps
        t = torch.tensor([e2e_ms], dtype=torch.float64, device=cdev if cdev is not None else "cpu")
        if world > 1:
            g = [torch.zeros_like(t) for _ in range(world)]
            dist.all_gather(g, t)
            e2e_max = max(float(x) for x in g)
        else:
            e2e_max = e2e_ms
        e2e = {"ms": e2e_max, "d2h": d2h // args.e2e_steps, "h2d": h2d // args.e2e_steps}

    if rank != 0:
        barrier()
        if world > 1:
            dist.destroy_process_group()
        return

    tot = corpus.combine(recs)
    max_ms = max(r["wall_ns"] for r in recs) / 1e6
    total_apps = tot["apps"]
    ms_step = max_ms / args.steps
    value = total_apps * args.steps / (max_ms / 1e3)
    peak, peak_src = measured_peak()
    achieved = alg / (fix_ns / 1e9) / 1e9 if fix_ns else 0.0
    traffic, traffic_wl = ncu_traffic(args.workload)
    parity = None
    if args.workload.startswith("corpus") and os.path.exists(CORPUS_CACHE):
        cache = json.load(open(CORPUS_CACHE))
        parity = corpus.check_digests(dig_all, dig_mask, cache["apps"]) if \
            cache.get("gen_version") == __import__("synth").generator.GEN_VERSION else {"stale_cache": True}
    pct = lambda xs, q: float(np.percentile(np.asarray(xs), q)) if xs else None
    line = {
        "metric": METRIC, "value": value, "unit": "apps/s", "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms_step,
        "higher_is_better": True, "scaling": scaling, "vs_baseline": None, "dtype": "u64",
        "data": "synthetic (seeded generator, Android-app-shaped ICFGs)",
        "config": {**desc, "batches_per_rank": [len(b) for b in plan.batches],
                   "nodes_rank0": nodes, "input_bytes_rank0": shard.input_bytes,
                   "l2": "fact stores > L2 (126 MB) per batch; re-zeroed each build",
                   "parallelism": f"apps sharded over {world} GPU(s), no data-path collective"},
        "ms_per_app": ms_step / (total_apps / world),
        "node_visits_per_s": tot["visits"] * args.steps / (max_ms / 1e3),
        "app_ms_rank0": {"p50": pct(app_ms, 50), "p90": pct(app_ms, 90), "p99": pct(app_ms, 99),
                         "max": max(app_ms) if app_ms else None,
                         "note": "an app's share of its batch's build time (apps of a batch share rounds), by node fraction"},
        "batch_ms_rank0": {"n": len(batch_ms), "sum": sum(batch_ms), "max": max(batch_ms),
                           "wide": sum(ms for b, ms in zip(my_batches, batch_ms) if plan.wide[b[0]])},
        "rounds_rank0": sum(s["rounds"] for s in stats),
        "fixpoint_ms_per_step_rank0": fix_ns / 1e6,
        "gpu_launches": launches * args.steps,
        "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                     "frac": achieved / peak, "traffic": traffic, "kernel": "k_fixpoint",
                     "bytes_model": "touched-word (SURVEY §8(d)), counted on the device by one untimed "
                                    "build of every batch with the counting instantiation; per launch = one "
                                    "step's k_fixpoint launches summed (achieved = bytes / their summed "
                                    "CUDA-event time; traffic = ncu DRAM bytes of the same launches)",
                     "alg_bytes_per_launch": alg, "dense_bytes_per_launch": dense,
                     "dense_achieved": dense / (fix_ns / 1e9) / 1e9 if fix_ns else 0.0,
                     "peak_source": peak_src, "traffic_workload": traffic_wl},
        "parity": parity,
        "clocks": clocks,
    }
    if e2e:
        line["e2e"] = {"value": total_apps / (e2e["ms"] / 1e3), "unit": "apps/s",
                       "h2d_bytes_per_step": e2e["h2d"], "d2h_bytes_per_step": e2e["d2h"],
                       "ms_per_step": e2e["ms"], "readback": args.e2e_readback,
                       "pipeline": "loader thread: gdroid_load_batch of batch i+1 (per-module host tables, raw "
                                   "descriptor arrays staged in pinned memory and uploaded, node/edge layout "
                                   "kernels, DESIGN.md §4.1) overlapped with the build of batch i; "
                                   "gdroid_read_batch_facts_async of batch i (pinned) overlapped with the build "
                                   "of batch i+1; one untimed warm-up pass sizes the buffers"}
    if not args.no_per_config and args.workload == "corpus1000":
        line["per_config"] = per_config_runs(local, stream.cuda_stream)
    if not args.no_cpu_baseline:
        import oracle
        oracle.build()
        P = host_threads()
        ids = oracle_sample_ids(plan, ORACLE_NODES_PER_CORE_S * P * args.cpu_seconds)
        sample_apps = [apps[i] if i in apps else make_app(i) for i in ids]
        if not sample_apps and not plan.wide[my_ids[0]]:
            ids, sample_apps = [my_ids[0]], [apps[my_ids[0]]]
    if not args.no_cpu_baseline and not sample_apps:
        line["cpu_baseline"] = {"value": None, "unit": "apps/s", "cores": P, "kind": "oracle",
                                "sample": "not timed: a worst-shaped app takes ~800 s of one core "
                                          "(tests/golden/oracle_digests.json records the oracle's time)"}
    elif not args.no_cpu_baseline:
        wall, osec, ovis, odig = oracle_pool(sample_apps, P)
        ok = sum(1 for i, d in zip(ids, odig) if d == int(dig_all[i]))   # vs the gathered GPU digests
        line["cpu_baseline"] = {
            "value": len(sample_apps) / wall, "unit": "apps/s", "cores": P, "kind": "oracle",
            "cpu_model": cpu_model(),
            "sample": f"{len(sample_apps)} apps ({sum(a.n_nodes for a in sample_apps)} nodes), a size-stratified "
                      f"sample of the workload's narrow apps, oracle on {P} host threads, {wall:.1f} s wall; "
                      f"the {sum(plan.wide)} worst-shaped apps are not in the timed sample",
            "node_visits_per_s": ovis / wall, "digests_equal_gpu": f"{ok}/{len(ids)}"}
    print(json.dumps(line), flush=True)
    barrier()
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
