"""Device search time of C4 query shards (1/2, 1/4, 1/8 of Q: what one rank
searches at N = 2, 4, 8), index resident, L2 flushed; the library's tile
size for each (DTS_TILE_Q forces one).  One JSON line per shard size."""
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
Dd = torch.from_numpy(c.D).cuda()
Qd = torch.from_numpy(c.Q).cuda()
idx = dts.build_index_device(Dd)
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
s = torch.cuda.current_stream()
for parts in (1, 2, 4, 8):
    m = len(c.Q) // parts
    Q = Qd[:m].contiguous()
    for _ in range(3):
        r, st = dts.search_device(idx, Q, c.d)
        r.free()
    ts = []
    for _ in range(10):
        flush.zero_()
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        e0.record(s)
        r, st = dts.search_device(idx, Q, c.d)
        e1.record(s)
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
        r.free()
    print(json.dumps({"tag": os.environ.get("DTS_TILE_Q", "auto"), "queries": m, "parts": parts,
                      "search_ms": statistics.median(ts), "tq": st["tile_queries"]}), flush=True)
