"""Time of the per-query work estimate (dts_query_costs_device, blocks of 256
queries) on C4 and its 1/8 share, index resident.  One JSON line each."""
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import paper_conf_ipps_gowanlockc15_b200 as dts  # noqa: E402
import synth  # noqa: E402

c = synth.make_config("C4")
idx = dts.build_index_device(torch.from_numpy(c.D).cuda())
Qd = torch.from_numpy(c.Q).cuda()
s = torch.cuda.current_stream()
for parts in (1, 8):
    Q = Qd[: len(c.Q) // parts].contiguous()
    ref = None
    ts = []
    for k in range(8):
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        e0.record(s)
        out = dts.query_costs_device(idx, Q, c.d, block=256, stride=int(os.environ.get("STRIDE", "1")))
        e1.record(s)
        torch.cuda.synchronize()
        if k >= 2:
            ts.append(e0.elapsed_time(e1))
        ref = int(out.sum())
    r, st = dts.search_device(idx, Q, c.d)
    r.free()
    print(json.dumps({"queries": len(Q), "costs_ms": statistics.median(ts), "sum": ref,
                      "search_candidates": st["candidates"]}), flush=True)
