"""Output-heavy search points (device search vs its pass-1
time): device search time (CUDA events, median of --reps after warm-ups,
index and Q resident) and the library's phase times.  One JSON line each.

    python scripts/heavy_points.py [--points C2:8 S2:1 C2:2]
"""
import argparse
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import paper_conf_ipps_gowanlockc15_b200 as dts  # noqa: E402
import synth  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--points", nargs="+", default=["C2:8", "S2:1", "C2:2"])
ap.add_argument("--reps", type=int, default=5)
ap.add_argument("--method", default="grid")
ap.add_argument("--no-hint", action="store_true", help="grid sized without d_hint = d")
a = ap.parse_args()
cache = {}
for pt in a.points:
    name, d = pt.split(":")
    d = float(d)
    key = (name, None if a.no_hint else d)
    if key not in cache:
        for v in cache.values():
            v[2].free()
        cache.clear()
        torch.cuda.empty_cache()
        c = synth.make_config(name)
        Dd = torch.from_numpy(c.D).cuda()
        Qd = torch.from_numpy(c.Q).cuda()
        # as scripts/sweep.py: the grid sized for the d searched (d_hint = d)
        cache[key] = (c, Qd, dts.build_index_device(Dd, method=a.method,
                                                    d_hint=0.0 if a.no_hint else d), Dd)
    c, Qd, idx, _ = cache[key]
    s = torch.cuda.current_stream()
    for _ in range(2):
        r, st = dts.search_device(idx, Qd, d, stream=s, time_kernels=True)
        r.free()
    ts, sts = [], []
    for _ in range(a.reps):
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        e0.record(s)
        r, st = dts.search_device(idx, Qd, d, stream=s, time_kernels=True)
        e1.record(s)
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
        sts.append(st)
        n = r.count
        r.free()
    ms = statistics.median(ts)
    ph = {k: statistics.median(x[k] for x in sts)
          for k in ("ms_prep", "ms_count", "ms_scan", "ms_scatter", "ms_canon")}
    print(json.dumps({"config": name, "d": d, "method": a.method, "search_ms": ms,
                      "phases_ms": ph, "ratio_to_pass1": ms / ph["ms_count"],
                      "results": n, "candidates": sts[-1]["candidates"],
                      "max_per_query": sts[-1]["max_results_per_query"]}), flush=True)
