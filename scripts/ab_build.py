"""A/B timing of the index build: the C4 (or --config) index built --reps
times on the device (L2 flushed before each), median of the library's phase
times (in-library CUDA events) and of the whole build (events around the
call).  One JSON line.

    DTS_LIB=ab/libdts_x.so python scripts/ab_build.py --config C4
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
ap.add_argument("--config", default="C4")
ap.add_argument("--reps", type=int, default=10)
ap.add_argument("--tag", default=os.environ.get("DTS_LIB", "tree"))
a = ap.parse_args()
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
c = synth.make_config(a.config)
Dd = torch.from_numpy(c.D).cuda()
s = torch.cuda.current_stream()
for _ in range(2):
    dts.build_index_device(Dd).free()
ts, ph = [], []
for _ in range(a.reps):
    flush.zero_()
    e0 = torch.cuda.Event(enable_timing=True)
    e1 = torch.cuda.Event(enable_timing=True)
    e0.record(s)
    idx = dts.build_index_device(Dd)
    e1.record(s)
    torch.cuda.synchronize()
    ts.append(e0.elapsed_time(e1))
    ph.append(idx.info()["ms_phase"])
    idx.free()
print(json.dumps({"lib": a.tag, "config": a.config, "build_ms": statistics.median(ts),
                  "phases": [statistics.median(p[i] for p in ph) for i in range(len(ph[0]))]}),
      flush=True)
