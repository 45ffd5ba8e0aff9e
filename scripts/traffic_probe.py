"""One search of a bench workload, for `ncu -k regex:k_wtile_count -c 1`
(bench.py measure_traffic): index built, then one device search with the
bench's launch configuration.  Prints nothing on success."""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import paper_conf_ipps_gowanlockc15_b200 as dts  # noqa: E402
import synth  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="C4")
ap.add_argument("--d", type=float, default=None)
ap.add_argument("--warm", type=int, default=0, help="untimed searches before the profiled one")
a = ap.parse_args()
c = synth.make_config(a.config)
d = a.d if a.d is not None else c.d
Dd = torch.from_numpy(c.D).cuda()
Qd = torch.from_numpy(c.Q).cuda()
idx = dts.build_index_device(Dd)
for _ in range(a.warm):
    r, _ = dts.search_device(idx, Qd, d)
    r.free()
torch.cuda.synchronize()
# only the search is profiled under `ncu --profile-from-start off`
torch.cuda.profiler.start()
res, _ = dts.search_device(idx, Qd, d)
torch.cuda.synchronize()
torch.cuda.profiler.stop()
res.free()
idx.free()
