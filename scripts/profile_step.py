"""Run W warm + K measured steps of the bench workload (for ncu launch lists
and full captures; numbers printed under a profiler are never bench values)."""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import synth  # noqa: E402
import paper_conf_ipps_gowanlockc15_b200 as dts  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="C4")
ap.add_argument("--steps", type=int, default=1)
ap.add_argument("--warmup", type=int, default=1)
ap.add_argument("--d", type=float, default=None)
a = ap.parse_args()
cfg = synth.make_config(a.config)
d = a.d if a.d is not None else cfg.d
Dd = torch.from_numpy(cfg.D).cuda()
Qd = torch.from_numpy(cfg.Q).cuda()
s = torch.cuda.current_stream()
for i in range(a.warmup + a.steps):
    idx = dts.build_index_device(Dd, stream=s)
    res, st = dts.search_device(idx, Qd, d, stream=s, time_kernels=True)
    print(i, res.count, st, idx.info(), flush=True)
    res.free()
    idx.free()
print("launches", dts.kernel_launches())
