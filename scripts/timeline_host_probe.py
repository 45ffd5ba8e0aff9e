"""GPU timeline of one host-API search (dts_search: pinned host Q -> pinned
host results, index resident) through CUPTI (torch.profiler): every copy and
kernel with its stream, start and duration, to see how the query-chunk
pipeline overlaps H2D, search and D2H.

    python scripts/timeline_host_probe.py [C4]
"""
import json
import os
import sys
import tempfile

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402
from torch.profiler import ProfilerActivity, profile  # noqa: E402

import paper_conf_ipps_gowanlockc15_b200 as dts  # noqa: E402
import synth  # noqa: E402

c = synth.make_config(sys.argv[1] if len(sys.argv) > 1 else "C4")
D = torch.from_numpy(c.D).pin_memory().numpy()
Q = torch.from_numpy(c.Q).pin_memory().numpy()
idx = dts.build_index(D)
for _ in range(3):
    r = dts.search(idx, Q, c.d)
    del r
torch.cuda.synchronize()
with profile(activities=[ProfilerActivity.CUDA]) as prof:
    r = dts.search(idx, Q, c.d)
    torch.cuda.synchronize()
path = tempfile.mktemp(suffix=".json")
prof.export_chrome_trace(path)
ev = json.load(open(path))["traceEvents"]
gpu = [e for e in ev if e.get("cat") in ("kernel", "gpu_memcpy", "gpu_memset")]
gpu.sort(key=lambda e: e["ts"])
t0 = gpu[0]["ts"]
print(f"{len(gpu)} GPU activities, last ends at {gpu[-1]['ts'] + gpu[-1]['dur'] - t0:.1f} us")
for e in gpu:
    a = e.get("args", {})
    nm = e["name"]
    if "Memcpy" in nm:
        nm += f" {a.get('bytes', 0) / 1e6:.1f} MB"
    print(f"  s{a.get('stream', '?'):>3} {e['ts'] - t0:8.1f} +{e['dur']:7.1f} us  {nm[:70]}")
