"""Per-phase device times of one config / method / d (diagnostics)."""
import argparse
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import paper_conf_ipps_gowanlockc15_b200 as dts  # noqa: E402
import synth  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="S3")
ap.add_argument("--d", type=float, nargs="+", default=[0.01, 0.09])
ap.add_argument("--method", default="grid")
a = ap.parse_args()
c = synth.make_config(a.config)
Dd = torch.from_numpy(c.D).cuda()
Qd = torch.from_numpy(c.Q).cuda()
for d in a.d:
    idx = dts.build_index_device(Dd, method=a.method, d_hint=d)
    for rep in range(4):
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        res, st = dts.search_device(idx, Qd, d, time_kernels=True)
        torch.cuda.synchronize()
        t1 = time.perf_counter()
        print(f"d={d} rep={rep} wall={1e3*(t1-t0):.3f}ms", {k: round(v, 4) if isinstance(v, float) else v
                                                        for k, v in st.items()}, flush=True)
        res.free()
    print(idx.info(), flush=True)
    idx.free()
