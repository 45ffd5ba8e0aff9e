"""C4 with 0.01% injected long segments: search time
with the long segments filed as copies along their path, against plain C4,
and (optionally) with plain filing (DTS_OUTLIERS=0 in a child process; the
long segments then size every cell and stencil).  One JSON line per run.

    python scripts/outlier_bench.py [--plain]
"""
import argparse
import json
import os
import statistics
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ipps_gowanlockc15_b200 as dts  # noqa: E402
import synth  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--frac", type=float, default=1e-4)
ap.add_argument("--reps", type=int, default=10)
ap.add_argument("--plain", action="store_true", help="also time DTS_OUTLIERS=0 (child process)")
ap.add_argument("--child", action="store_true")
a = ap.parse_args()


def long_segments(n, seed):
    """n segments: 30 units of travel over 40 time steps through the galaxy
    region, random direction (every fourth along x, every fifth stationary)."""
    g = synth.rng(seed)
    L = np.zeros((n, 8))
    t0 = g.uniform(0.0, 152.0, n)
    p0 = g.uniform(-12.0, 12.0, (n, 3))
    p0[:, 2] = g.uniform(-1.0, 1.0, n)
    dirs = g.normal(0, 1, (n, 3))
    dirs[::4] = [1.0, 0.0, 0.0]
    dirs /= np.linalg.norm(dirs, axis=1)[:, None]
    length = np.full(n, 30.0)
    length[1::5] = 0.0
    L[:, 0], L[:, 4] = t0, t0 + 40.0
    L[:, 1:4] = p0
    L[:, 5:8] = p0 + dirs * length[:, None]
    return L


def timed(idx, Qd, d, reps):
    s = torch.cuda.current_stream()
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    for _ in range(3):
        r, _ = dts.search_device(idx, Qd, d, stream=s)
        r.free()
    ts, st = [], None
    for _ in range(reps):
        flush.zero_()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s)
        r, st = dts.search_device(idx, Qd, d, stream=s, time_kernels=True)
        e1.record(s)
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
        n = r.count
        r.free()
    return statistics.median(ts), st, n


c = synth.make_config("C4")
k = max(1, int(round(a.frac * c.D.shape[0])))
D = np.ascontiguousarray(np.concatenate([c.D, long_segments(k, 77)]))
Qd = torch.from_numpy(c.Q).cuda()
rows = []
for name, DD in ([("C4+long", D)] if a.child else [("C4", c.D), ("C4+long", D)]):
    idx = dts.build_index_device(torch.from_numpy(DD).cuda())
    inf = idx.info()
    ms, st, n = timed(idx, Qd, c.d, a.reps)
    rows.append({"data": name, "outliers_env": os.environ.get("DTS_OUTLIERS", "1"),
                 "n_entries": int(DD.shape[0]), "long_segments": k if name != "C4" else 0,
                 "search_ms": ms, "count_pass_ms": st["ms_count"], "results": n,
                 "candidates": st["candidates"], "outlier_rows": inf["outlier_rows"],
                 "outlier_copies": inf["outlier_copies"], "grid": inf["grid"],
                 "max_extent": inf["max_extent"], "ms_build": inf["ms_build"]})
    idx.free()
if not a.child and len(rows) == 2:
    rows[1]["regression_vs_plain_C4"] = rows[1]["search_ms"] / rows[0]["search_ms"] - 1.0
for r in rows:
    print(json.dumps(r), flush=True)
if a.plain and not a.child:
    out = subprocess.run([sys.executable, __file__, "--child", "--reps", "3", "--frac", str(a.frac)],
                         env={**os.environ, "DTS_OUTLIERS": "0"}, capture_output=True, text=True,
                         timeout=900)
    sys.stdout.write(out.stdout)
    sys.stderr.write(out.stderr[-2000:])
