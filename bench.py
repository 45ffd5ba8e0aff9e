#!/usr/bin/env python
"""Benchmark of the distance threshold search hot path (BASELINE.json metric:
search time and query-segments/s at 1/2/4/8 B200, % HBM roofline).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config C4] [--impl reference]

A step = one pass of the whole hot path over the
workload: index build over the resident entry set D, query prep, both fused
candidate-streaming + refinement passes, the exact-offset scan, canonical
ordering.  `value` is device-timed throughput with inputs already in HBM;
`e2e` is the same metric through the C ABI's host entry points (pinned host
D and Q copied in, results copied out every step).  Multi-GPU (torchrun):
weak scaling, every rank searches its own 1M-query set against the replicated
D; the only collective is an all_gather of the per-rank result counts (global
offsets).  Rank 0 prints one JSON line.

The oracle (oracle/, test infrastructure) runs only in the cpu_baseline leg
(rank 0, N=1) and in --impl reference.
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

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)

import synth  # noqa: E402

METRIC = "query-segments/s (search step incl. index build; BASELINE: search time and q-seg/s at 1/2/4/8 B200, % HBM roofline)"
UNIT = "query-segments/s"
WORKLOADS = {
    "C4": "galaxy-shaped synthetic at scale: 20,132,736 entry segments (104,858 stellar-orbit "
          "trajectories x 192 steps), 1,000,128 query segments per rank (5,209 trajectories "
          "sampled from D), d=0.005 (BASELINE.json configs[4])",
    "C1": "galaxy-shaped synthetic: 1,048,512 entry segments, 9,984 query segments, d=0.005 "
          "(BASELINE.json configs[1])",
    "C2": "uniform dense random walks: 4,194,432 entries, 100,032 queries (configs[2])",
    "C3": "uniform sparse long-span random walks: 3,990,000 entries, 99,750 queries (configs[3])",
}


def _env_int(k, default):
    try:
        return int(os.environ.get(k, default))
    except ValueError:
        return default


def load_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        j = json.load(open(p))
        return float(j["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled during the timed region."""

    def __init__(self, index: int):
        self.index = index
        self.rows = []
        self.proc = None
        self.thread = None

    def start(self):
        q = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
             "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
             "clocks_event_reasons.sw_power_cap")
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.index), f"--query-gpu={q}",
                 "--format=csv,noheader,nounits", "-lms", "100"],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        except OSError:
            self.proc = None
            return

        def reader():
            for line in self.proc.stdout:
                self.rows.append([x.strip() for x in line.split(",")])

        self.thread = threading.Thread(target=reader, daemon=True)
        self.thread.start()

    def stop(self):
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except subprocess.TimeoutExpired:
            self.proc.kill()
        if self.thread:
            self.thread.join(timeout=2)
        sm, mx, reasons = [], None, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for r in self.rows:
            try:
                sm.append(float(r[0]))
                mx = float(r[1])
                for k, nm in enumerate(names):
                    if r[3 + k].lower().startswith("active"):
                        reasons.add(nm)
            except (ValueError, IndexError):
                continue
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": mx,
                "reasons": sorted(reasons), "samples": len(sm)}


def host_cores():
    try:
        return len(os.sched_getaffinity(0))
    except AttributeError:
        return os.cpu_count() or 1


def oracle_rate(cfg, seconds: float, seed: int):
    """Oracle (as it stands) on a bounded sample of the workload's queries:
    brute force of each sampled query against all of D, one single-threaded
    oracle instance per host core.  Returns (q-seg/s, cores, sample text)."""
    import oracle
    oracle.build()
    cores = host_cores()
    g = synth.rng(seed)
    t = time.perf_counter()
    oracle.search_queries(cfg.D, cfg.Q, [int(g.integers(cfg.Q.shape[0]))], cfg.d)
    t1 = max(time.perf_counter() - t, 1e-4)               # one query, one core
    nsample = int(max(cores, min(20000, cores * max(1, round(seconds / t1)))))
    qs = np.sort(g.choice(cfg.Q.shape[0], size=min(nsample, cfg.Q.shape[0]), replace=False))
    t = time.perf_counter()
    oracle.search_queries(cfg.D, cfg.Q, qs, cfg.d, threads=cores)
    el = time.perf_counter() - t
    sample = (f"{qs.size} query segments sampled uniformly (seed {seed}) from the workload's "
              f"{cfg.Q.shape[0]}, each brute-forced against all {cfg.D.shape[0]} entries; "
              f"{el:.1f} s wall on {cores} threads")
    return qs.size / el, cores, sample


def run_reference(args):
    rank = _env_int("RANK", 0)
    if rank != 0:
        return 0
    cfg = synth.make_config(args.config)
    cores = host_cores()
    times = []
    last_sample = ""
    # the whole --steps K --warmup W run stays within ~--ref-budget-seconds
    per_step_s = max(0.5, min(args.ref_step_seconds,
                              args.ref_budget_seconds / max(1, args.steps + args.warmup)))
    for i in range(args.warmup + args.steps):
        v, cores, sample = oracle_rate(cfg, per_step_s, seed=500 + i)
        if i >= args.warmup:
            times.append(v)
            last_sample = sample
    value = statistics.median(times)
    line = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": UNIT,
        "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": 1e3 * cfg.Q.shape[0] / value, "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": {"workload": WORKLOADS.get(args.config, args.config), "name": args.config,
                   "n_entries": int(cfg.D.shape[0]), "n_queries": int(cfg.Q.shape[0]),
                   "d": cfg.d},
        "cpu_baseline": {"value": value, "unit": UNIT, "cores": cores, "kind": "oracle",
                         "sample": "per step: " + last_sample},
        "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
        "note": "plain single-threaded C brute force (oracle/), one instance per host core; "
                "ms_per_step extrapolates the sampled rate to the full query set",
    }
    print(json.dumps(line), flush=True)
    return 0


def run_own(args):
    import torch
    import torch.distributed as dist

    world = _env_int("WORLD_SIZE", 1)
    rank = _env_int("RANK", 0)
    local = _env_int("LOCAL_RANK", 0)
    # one process per GPU; DTS_DIST_BACKEND=gloo (with more ranks than GPUs:
    # device = local rank mod GPU count) only exercises the multi-rank code
    # path on a one-GPU box -- its timings are not scaling numbers
    backend = os.environ.get("DTS_DIST_BACKEND", "nccl")
    local = local % max(1, torch.cuda.device_count())
    torch.cuda.set_device(local)
    if world > 1:
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        else:
            dist.init_process_group(backend)
    dev = torch.device("cuda", local)

    import paper_conf_ipps_gowanlockc15_b200 as dts
    from paper_conf_ipps_gowanlockc15_b200 import dist as dts_dist
    dts.load()

    cfg = synth.make_config(args.config, rank=rank)
    d = args.d if args.d is not None else cfg.d
    n, nq = cfg.D.shape[0], cfg.Q.shape[0]
    D_pin = torch.from_numpy(cfg.D).pin_memory()
    Q_pin = torch.from_numpy(cfg.Q).pin_memory()
    D_dev = D_pin.to(dev, non_blocking=False)
    Q_dev = Q_pin.to(dev, non_blocking=False)
    stream = torch.cuda.current_stream(dev)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)   # > 126 MB L2

    def step():
        """The hot path of one step: returns when its results are on the
        device (the library syncs for the result count)."""
        idx = dts.build_index_device(D_dev, device=local, stream=stream)
        res, st = dts.search_device(idx, Q_dev, d, stream=stream, time_kernels=True)
        if world > 1:
            dts_dist.global_offset(res.count, rank, world)
        return idx, res, st

    def finish(idx, res, st, stats_out=None):
        """Bookkeeping after the timed region of a step: phase times, frees."""
        if stats_out is not None:
            inf = idx.info()
            st["ms_build"] = inf["ms_build"]
            st["ms_phase"] = list(inf["ms_phase"])
            st["index"] = inf
            stats_out.append(st)
        cnt = res.count
        res.free()
        idx.free()
        return cnt

    for _ in range(max(args.warmup, 0)):
        finish(*step())
    torch.cuda.synchronize(dev)
    if world > 1:
        dist.barrier()

    # ---- timed region: per-step CUDA events on the launching stream, L2
    #      flushed between steps (outside the events)
    clocks = ClockSampler(local)
    clocks.start()
    launches0 = dts.kernel_launches()
    evs = []
    stats = []
    torch.cuda.synchronize(dev)
    if world > 1:
        dist.barrier()
    wall0 = time.perf_counter()
    results = 0
    for _ in range(args.steps):
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        out = step()
        e1.record(stream)
        evs.append((e0, e1))
        flush.zero_()
        results = finish(*out, stats_out=stats)
    torch.cuda.synchronize(dev)
    wall = time.perf_counter() - wall0
    if world > 1:
        dist.barrier()
    launches = dts.kernel_launches() - launches0
    clk = clocks.stop()
    step_ms = [a.elapsed_time(b) for a, b in evs]
    total_ms = sum(step_ms)
    if world > 1:
        t = torch.tensor([total_ms], device=dev if backend == "nccl" else "cpu",
                         dtype=torch.float64)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        total_ms = float(t.item())
    ms_per_step = total_ms / args.steps
    value = world * nq / (ms_per_step * 1e-3)

    # ---- per-kernel rooflines (CUDA events in-lib, on the launching stream):
    #      algorithmic bytes per launch / mean event time
    peak, peak_src = load_peaks()
    st0 = stats[-1]
    ms_count = statistics.mean(s["ms_count"] for s in stats)
    ms_scatter = statistics.mean(s["ms_scatter"] for s in stats)
    ms_build = statistics.mean(s["ms_build"] for s in stats)
    ph = [statistics.mean(s["ms_phase"][i] for s in stats) for i in range(5)]
    inf = st0["index"]
    ncell_key = inf["bins"] * inf["grid"][0] * inf["grid"][1] * inf["grid"][2]
    kbits = max(1, int(ncell_key - 1).bit_length())
    npass = (kbits + 7) // 8                 # the library's digit plan: 9-bit digits
    if npass > 1 and kbits <= 9 * (npass - 1):   # where they save a pass
        npass -= 1
    ncells = inf["cells"]
    alg_bytes = st0["candidates"] * 64 + nq * (64 + 4) + st0["cell_lookups"] * 64
    traffic_all = {}
    tf = os.path.join(ROOT, "profiles", "traffic.json")
    if os.path.exists(tf):
        try:
            traffic_all = json.load(open(tf)).get(args.config, {})
        except (ValueError, AttributeError):
            traffic_all = {}
    kernels = [
        # name, ms per launch-group, algorithmic bytes, model
        ("k_wtile_count", ms_count, alg_bytes,
         "64 B per candidate + 68 B per query + 64 B per hash-bucket probe"),
        ("k_onesweep (entry sort)", ph[2],
         (0 if inf.get("build_flags", 0) & 1 else n * 8) + npass * n * 16,
         f"{npass} passes x (8 B read + 8 B write) per key"
         + ("" if inf.get("build_flags", 0) & 1 else " + 8 B/key histogram read")
         + "; issue/latency-bound, not HBM-bound (DRAM ~15% busy): CUB DeviceRadixSort "
           "takes 1.09 ms on the same shape (profiles/r01d_cub_sort.txt)"),
        ("k_gather_cells", ph[3], n * (8 + 64 + 68),
         "8 B sorted key + 64 B record read + 68 B record/id write per entry"),
        ("k_insert_blocks_lane" if inf.get("hash_kind", 0) == 1 else "k_insert_tiled", ph[4],
         n * 8 + inf.get("hash_items", ncells) * (32 if inf.get("hash_kind", 0) == 1 else 16),
         "8 B key per entry + one slot per hash item (32 B per 8-key block, or 16 B per cell); "
         "phase includes the table memset"),
    ]
    if inf.get("build_flags", 0) & 1:
        kernels += [
            ("k_bounds_keys", ph[1], n * (64 + 8), "64 B record read + 8 B key write per entry "
             "(exact bounds, packed keys and all sort-pass digit counts in one read)"),
            ("k_bounds_sample", ph[0], 65536 * 64, "64 B per sampled entry (2^16 sample; "
             "phase includes the host read-back)"),
        ]
    else:
        kernels += [
            ("k_bounds", ph[0], n * 64, "64 B record read per entry"),
            ("k_keys", ph[1], n * (64 + 8), "64 B record read + 8 B key write per entry "
             "(phase includes the host read-back of the bounds)"),
        ]
    kern = []
    for name, ms, by, model in kernels:
        a_gbs = by / (ms * 1e-3) / 1e9 if ms > 0 else None
        kern.append({"kernel": name, "ms": ms, "bytes": int(by), "achieved_gbs": a_gbs,
                     "frac": (a_gbs / peak) if a_gbs else None,
                     "traffic": traffic_all.get(name.split()[0]), "bytes_model": model})
    dom = max(kern, key=lambda k: k["ms"])
    achieved = alg_bytes / (ms_count * 1e-3) / 1e9
    traffic = traffic_all.get("k_wtile_count")

    # ---- e2e through the C ABI host entry points (pinned host buffers)
    e2e_val = None
    e2e_search = None
    h2d = (n + nq) * 64
    d2h = results * 24
    if rank == 0 or world > 1:
        D_np = D_pin.numpy()
        Q_np = Q_pin.numpy()
        ts = []
        ts_search = []
        for i in range(max(1, args.e2e_steps) + 1):
            torch.cuda.synchronize(dev)
            t0 = time.perf_counter()
            idx = dts.build_index(D_np, device=local)
            t1 = time.perf_counter()
            res = dts.search(idx, Q_np, d)
            t2 = time.perf_counter()
            if i > 0:
                ts.append(t2 - t0)
                ts_search.append(t2 - t1)
            d2h = res.nbytes
            idx.free()
            del res
        e2e_val = world * nq / statistics.median(ts)
        e2e_search = world * nq / statistics.median(ts_search)

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        v, cores, sample = oracle_rate(cfg, args.cpu_seconds, seed=42)
        cpu = {"value": v, "unit": UNIT, "cores": cores, "kind": "oracle", "sample": sample}

    if rank == 0:
        line = {
            "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms_per_step,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None,
            "dtype": "f64", "data": "synthetic",
            "config": {"workload": WORKLOADS.get(args.config, args.config), "name": args.config,
                       "n_entries": int(n), "n_queries_per_rank": int(nq), "d": d,
                       "step": "index build + query prep + count pass + scan + scatter pass + "
                               "canonical sort (all SURVEY.md §8(a) rows), inputs resident in HBM",
                       "l2": "flushed between steps (256 MiB write outside the timed events)",
                       "parallelism": f"query-sharded x{world}, D replicated"},
            "phases_ms": {"build": ms_build, "build_bounds": ph[0], "build_keys": ph[1],
                          "build_sort": ph[2], "build_gather": ph[3], "build_insert": ph[4],
                          "prep": statistics.mean(s["ms_prep"] for s in stats),
                          "count_pass": ms_count, "scan": statistics.mean(s["ms_scan"] for s in stats),
                          "scatter_pass": ms_scatter,
                          "canon": statistics.mean(s["ms_canon"] for s in stats)},
            "search_only": {"value": world * nq / ((ms_per_step - ms_build) * 1e-3), "unit": UNIT,
                            "note": "step minus index build (the paper's response time excludes "
                                    "the build, P:L135)"},
            "work": {"candidates_per_pass": st0["candidates"], "cell_lookups": st0["cell_lookups"],
                     "results_per_rank": results},
            "roofline": {"bound": "hbm", "kernel": dom["kernel"], "achieved": dom["achieved_gbs"],
                         "peak": peak, "unit": "GB/s", "frac": dom["frac"],
                         "traffic": dom["traffic"], "peak_source": peak_src,
                         "algorithmic_bytes": dom["bytes"], "ms": dom["ms"],
                         "bytes_model": dom["bytes_model"],
                         "note": "dominant kernel = largest device time of one step "
                                 "(per-phase CUDA events); all kernels in roofline_kernels"},
            "roofline_kernels": kern,
            "roofline_search": {"bound": "hbm", "kernel": "k_wtile_count (pass 1: fused candidate "
                                "streaming + fp64 refine)", "achieved": achieved, "peak": peak,
                                "unit": "GB/s", "frac": achieved / peak, "traffic": traffic,
                                "algorithmic_bytes": alg_bytes},
            "clocks": clk,
            "gpu_launches": int(launches),
            "e2e": {"value": e2e_val, "unit": UNIT, "h2d_bytes_per_step": int(h2d),
                    "d2h_bytes_per_step": int(d2h),
                    "search_only_value": e2e_search,
                    "note": "dts_build_index(host D) + dts_search(host Q) -> host results, "
                            "wall clock, median of steps"},
            "wall_s_timed": wall,
        }
        if cpu is not None:
            line["cpu_baseline"] = cpu
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()
    return 0


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=100)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default="C4")
    ap.add_argument("--d", type=float, default=None)
    ap.add_argument("--impl", default="own", choices=["own", "reference"])
    ap.add_argument("--e2e-steps", type=int, default=3)
    ap.add_argument("--cpu-seconds", type=float, default=15.0)
    ap.add_argument("--ref-step-seconds", type=float, default=8.0)
    ap.add_argument("--ref-budget-seconds", type=float, default=150.0,
                    help="reference arm: oracle seconds for the whole run (per-step samples "
                         "shrink with --steps + --warmup)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    args = ap.parse_args()
    if args.warmup < 3:
        args.warmup = 3
    if args.impl == "reference":
        return run_reference(args)
    return run_own(args)


if __name__ == "__main__":
    sys.exit(main())
