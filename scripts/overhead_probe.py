"""Fixed per-call cost of a search: device step time (events around the
call, L2 flushed) of the C4 search with and without the library's phase
events, and of searches of 16 / 1024 queries of the same index; host wall
time of each call.  One JSON line per point."""
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

c = synth.make_config(os.environ.get("CFG", "C4"))
Dd = torch.from_numpy(c.D).cuda()
Qd = torch.from_numpy(c.Q).cuda()
idx = dts.build_index_device(Dd)
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
s = torch.cuda.current_stream()
for nq, tk in ((len(c.Q), False), (len(c.Q), True), (len(c.Q), "defer"), (16, False), (16, True), (16, "defer"), (1024, False), (65536, False))[: int(os.environ.get("NPTS", "8"))]:
    Q = Qd[:nq].contiguous()
    for _ in range(3):
        r, _st = dts.search_device(idx, Q, c.d, stream=s, time_kernels=tk)
        r.free()
    ev, wall = [], []
    for _ in range(20):
        flush.zero_()
        torch.cuda.synchronize()
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        e0.record(s)
        t0 = time.perf_counter()
        r, st = dts.search_device(idx, Q, c.d, stream=s, time_kernels=tk)
        t1 = time.perf_counter()
        e1.record(s)
        torch.cuda.synchronize()
        ev.append(e0.elapsed_time(e1))
        wall.append((t1 - t0) * 1e3)
        r.free()
    print(json.dumps({"nq": nq, "time_kernels": tk, "step_ms": statistics.median(ev),
                      "wall_ms": statistics.median(wall),
                      "phases": {k: st.get(k) for k in ("ms_prep", "ms_count", "ms_scan", "ms_scatter", "ms_canon")}}),
          flush=True)
