"""A/B timing of the search (index resident): for each point, device search
time (CUDA events, median of --reps after warm-ups, L2 flushed between reps)
and the library's phase times.  The library is the one DTS_LIB names (else
the in-tree build).  One JSON line per point.

    DTS_LIB=ab/libdts_base.so python scripts/ab_search.py --points C4:0.005 C2:2
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
ap.add_argument("--points", nargs="+", default=["C4:0.005", "C4:0.02", "C2:2", "C1:0.005"])
ap.add_argument("--reps", type=int, default=20)
ap.add_argument("--tag", default=os.environ.get("DTS_LIB", "tree"))
a = ap.parse_args()
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
cache = {}
for pt in a.points:
    name, d = pt.split(":")
    d = float(d)
    hint = 0.0 if name == "C4" else d
    key = (name, hint)
    if key not in cache:
        for v in cache.values():
            v[1].free()
        cache.clear()
        c = synth.make_config(name)
        Dd = torch.from_numpy(c.D).cuda()
        Qd = torch.from_numpy(c.Q).cuda()
        # build twice (the first maps fresh pages); phases of the second
        i0 = dts.build_index_device(Dd, d_hint=hint)
        i0.info()
        i0.free()
        cache[key] = (Qd, dts.build_index_device(Dd, d_hint=hint), Dd)
    Qd, idx, _ = cache[key]
    binf = idx.info()
    s = torch.cuda.current_stream()
    for _ in range(3):
        r, st = dts.search_device(idx, Qd, d, stream=s, time_kernels=True)
        r.free()
    ts, sts = [], []
    for _ in range(a.reps):
        flush.zero_()
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
    print(json.dumps({"lib": a.tag, "config": name, "d": d, "search_ms": statistics.median(ts),
                      "count_ms": statistics.median(x["ms_count"] for x in sts),
                      "prep_ms": statistics.median(x["ms_prep"] for x in sts),
                      "emit_ms": statistics.median(x["ms_scatter"] for x in sts),
                      "canon_ms": statistics.median(x["ms_canon"] for x in sts), "tq": sts[-1].get("tile_queries"), "work": sts[-1].get("work_estimate"),
                      "results": n, "candidates": sts[-1]["candidates"],
                      "build_ms": binf["ms_build"], "build_phases": binf["ms_phase"],
                      "hash_bytes": binf["hash_bytes"]}), flush=True)
