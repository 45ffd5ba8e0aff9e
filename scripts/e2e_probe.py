"""End-to-end host-API search timing (dts_search: pinned host Q -> pinned host
results, index resident) for a few DTS_Q_CHUNK settings, each in its own
process (the knob is read once).  Prints one JSON line per setting."""
import json
import os
import statistics
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CODE = r'''
import sys, time, statistics, json
sys.path.insert(0, %r)
import torch, synth, paper_conf_ipps_gowanlockc15_b200 as dts
c = synth.make_config(%r)
D = torch.from_numpy(c.D).pin_memory().numpy()
Q = torch.from_numpy(c.Q).pin_memory().numpy()
idx = dts.build_index(D)
ts = []
for i in range(8):
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    r = dts.search(idx, Q, c.d)
    ts.append(time.perf_counter() - t0)
    n = r.shape[0]
    del r
print(json.dumps({"ms": 1e3 * statistics.median(ts[2:]), "min_ms": 1e3 * min(ts[2:]), "results": n}))
'''
cfg = sys.argv[1] if len(sys.argv) > 1 else "C4"
for chunk in sys.argv[2:] or ["0", "131072", "262144", "500064"]:
    env = dict(os.environ, DTS_Q_CHUNK=chunk)
    out = subprocess.run([sys.executable, "-c", CODE % (ROOT, cfg)], env=env, capture_output=True,
                         text=True, timeout=600)
    line = out.stdout.strip().splitlines()[-1] if out.stdout.strip() else out.stderr[-300:]
    print(json.dumps({"config": cfg, "chunk": int(chunk), "result": line}), flush=True)
