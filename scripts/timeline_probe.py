"""GPU timeline of a few searches (CUPTI activity records through
torch.profiler): each kernel / memcpy / memset of the library with its start
and duration relative to the search's first GPU activity, and the idle gaps
between them.  Prints one block per search size.

    python scripts/timeline_probe.py [C4]
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
Dd = torch.from_numpy(c.D).cuda()
Qd = torch.from_numpy(c.Q).cuda()
idx = dts.build_index_device(Dd)
for nq in (16, 65536, len(c.Q)):
    Q = Qd[:nq].contiguous()
    for _ in range(3):
        r, _ = dts.search_device(idx, Q, c.d)
        r.free()
    torch.cuda.synchronize()
    with profile(activities=[ProfilerActivity.CPU, ProfilerActivity.CUDA]) as prof:
        r, _ = dts.search_device(idx, Q, c.d)
        torch.cuda.synchronize()
    r.free()
    path = tempfile.mktemp(suffix=".json")
    prof.export_chrome_trace(path)
    ev = json.load(open(path))["traceEvents"]
    gpu = [e for e in ev if e.get("cat") in ("kernel", "gpu_memcpy", "gpu_memset")]
    gpu.sort(key=lambda e: e["ts"])
    if not gpu:
        print("no GPU activity recorded")
        continue
    t0 = gpu[0]["ts"]
    print(f"== nq {nq}: {len(gpu)} GPU activities, first at 0, last ends at "
          f"{gpu[-1]['ts'] + gpu[-1]['dur'] - t0:.1f} us")
    end = t0
    for e in gpu:
        gap = e["ts"] - end
        print(f"  {e['ts'] - t0:8.1f} +{e['dur']:7.1f} us  gap {gap:6.1f}  {e['name'][:60]}")
        end = max(end, e["ts"] + e["dur"])
    cpu = [e for e in ev if e.get("cat") == "cuda_runtime"]
    if cpu:
        c0 = min(e["ts"] for e in cpu)
        print(f"  host runtime calls: {len(cpu)}, first at {c0 - t0:.1f} us (rel. first GPU op), "
              f"sum {sum(e['dur'] for e in cpu):.1f} us")
