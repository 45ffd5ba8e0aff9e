"""Method x distance sweep on one GPU.

For each config and each candidate generator (grid / temporal / subbin) and
each d: device search time (CUDA events, median of --reps after a warm-up,
index resident, Q resident), the paper's response time (host Q -> host
results through dts_search, wall clock, median of 3, index build excluded as
in P:L135), candidates refined, probes, results.  One JSON line per point.

    python scripts/sweep.py --configs C1 C2 C3 S1 S2 S3 --out gpurun_out/sweep.jsonl
"""
import argparse
import json
import os
import statistics
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import paper_conf_ipps_gowanlockc15_b200 as dts  # noqa: E402
import synth  # noqa: E402

PAPER_V = {"S1": 4, "S2": 16, "S3": 4, "C1": 16, "C4": 16, "C2": 4, "C3": 4}


def timed_search(idx, Qd, d, reps):
    """Median device time of uninstrumented searches; the phase times come
    from one more, instrumented, search."""
    s = torch.cuda.current_stream()
    res, st = dts.search_device(idx, Qd, d, stream=s, time_kernels=True)
    res.free()
    ts = []
    for _ in range(reps):
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        e0.record(s)
        res, _ = dts.search_device(idx, Qd, d, stream=s)
        e1.record(s)
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
        n = res.count
        res.free()
    return statistics.median(ts), st, n


def response_time(idx, Q, d):
    ts = []
    for _ in range(3):
        t0 = time.perf_counter()
        r = dts.search(idx, Q, d)
        ts.append(time.perf_counter() - t0)
        del r
    return statistics.median(ts)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--configs", nargs="+", default=["C1", "C2", "C3"])
    ap.add_argument("--methods", nargs="+", default=["grid", "temporal", "subbin"])
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--dmax", type=float, default=None,
                    help="skip distances above this (S2 at d = 5 has 7.5e9 results: 180 GB "
                         "of host memory)")
    ap.add_argument("--out", default=None)
    a = ap.parse_args()
    out = open(a.out, "a") if a.out else None
    for name in a.configs:
        c = synth.make_config(name)
        Dd = torch.from_numpy(c.D).cuda()
        Qd = torch.from_numpy(c.Q).cuda()
        for method in a.methods:
            built = {}
            for d in c.d_sweep:
                if a.dmax is not None and d > a.dmax:
                    continue
                key = d if method == "grid" else None
                if key not in built:
                    for k in list(built):
                        built.pop(k).free()
                    t0 = time.perf_counter()
                    idx = dts.build_index_device(
                        Dd, method=method, d_hint=(d if method == "grid" else 0.0),
                        subbins=PAPER_V.get(name, 16) if method == "subbin" else 0)
                    torch.cuda.synchronize()
                    built[key] = idx
                    build_s = time.perf_counter() - t0
                idx = built[key]
                try:
                    ms, st, nres = timed_search(idx, Qd, d, a.reps)
                except dts.DTSError as e:        # results exceed device memory
                    ms, st, nres = None, {"candidates": None, "cell_lookups": None,
                                          "ms_count": None, "ms_prep": None}, None
                    print(f"# device search skipped: {e}", flush=True)
                rt = response_time(idx, c.Q, d)
                if nres is None:
                    nres = int(dts.search(idx, c.Q, d).shape[0])
                rec = {"config": name, "method": method, "d": d, "n": int(c.D.shape[0]),
                       "nq": int(c.Q.shape[0]), "search_ms_device": ms,
                       "qseg_per_s_device": c.Q.shape[0] / (ms * 1e-3) if ms else None,
                       "response_time_s": rt, "qseg_per_s_response": c.Q.shape[0] / rt,
                       "results": nres, "candidates": st["candidates"],
                       "cell_probes": st["cell_lookups"], "ms_count_pass": st["ms_count"],
                       "ms_prep": st["ms_prep"], "build_s_wall": build_s,
                       "index": {k: v for k, v in idx.info().items()
                                 if k in ("bins", "cells", "grid", "subbins", "ms_build")}}
                line = json.dumps(rec)
                print(line, flush=True)
                if out:
                    out.write(line + "\n")
                    out.flush()
            for k in list(built):
                built.pop(k).free()
        del Dd, Qd
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
