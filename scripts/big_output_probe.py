"""Response time of an output-heavy host search (dts_search: host Q -> host
results), e.g. S2 at d = 1 (4.3e8 results, 10.4 GB), index resident.  One
JSON line."""
import json
import os
import statistics
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_ipps_gowanlockc15_b200 as dts  # noqa: E402
import synth  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "S2"
d = float(sys.argv[2]) if len(sys.argv) > 2 else 1.0
c = synth.make_config(name)
idx = dts.build_index(c.D, d_hint=d)
ts = []
n = 0
for _ in range(3):
    t0 = time.perf_counter()
    r = dts.search(idx, c.Q, d)
    ts.append(time.perf_counter() - t0)
    n = r.shape[0]
    chk = int(r["entry_id"][:: max(1, n // 1000)].sum())
    del r
print(json.dumps({"config": name, "d": d, "results": n, "response_s": ts,
                  "median_s": statistics.median(ts), "gb": n * 24 / 1e9, "chk": chk}), flush=True)
