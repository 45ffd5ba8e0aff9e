"""Small workloads through every kernel path, for compute-sanitizer
(memcheck / racecheck / synccheck)."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ipps_gowanlockc15_b200 as dts  # noqa: E402
import synth  # noqa: E402

c = synth.make_config("C0")
for method in ("grid", "temporal", "subbin"):
    idx = dts.build_index(c.D, method=method, entry_traj=c.etraj)
    for d in (0.0, 0.05, 0.3):
        dts.search(idx, c.Q, d)
    dts.search_ex(idx, c.Q, 0.2, query_traj=c.qtraj, exclude_same_trajectory=True)
    idx.free()
# heavy output (recompute + radix canonicalisation path)
g = np.random.default_rng(1)
D = np.zeros((1500, 8))
D[:, 4] = 1.0
D[:, 1:4] = g.uniform(0, 0.02, size=(1500, 3))
D[:, 5:8] = D[:, 1:4]
Q = D[:20].copy()
idx = dts.build_index(D)
r = dts.search(idx, Q, 0.05)
# device API, trajectory merge, canonicalise
Dd = torch.from_numpy(c.D).cuda()
Qd = torch.from_numpy(c.Q).cuda()
idx = dts.build_index_device(Dd)
res, _ = dts.search_device(idx, Qd, 0.2)
m = dts.merge_trajectories_device(res, torch.from_numpy(c.qtraj).cuda(),
                                  torch.from_numpy(c.etraj).cuda())
t = res.tensor().clone()
dts.canonicalize_device(t)
print("sanitize workload ok", r.shape[0], res.count, m.count, flush=True)
# crowded hash blocks (> 65,535 entries in one 8-cell block, warp-path
# inserts) plus one long segment (coarse cells, multi-row stencils)
D, Q = synth.crowded(5)
D = np.concatenate([D, [[0.0, 0.05, 0.5, 0.5, 1.0, 0.95, 0.52, 0.5]]])
idx = dts.build_index(D)
r2 = dts.search(idx, Q, 0.01)
idx.free()
# a multi-tile onesweep sort (look-back across tiles) and the cost kernel
c1 = synth.make_config("C1", scale=0.1)
idx = dts.build_index_device(torch.from_numpy(c1.D).cuda())
Q1 = torch.from_numpy(c1.Q).cuda()
res1, _ = dts.search_device(idx, Q1, 0.02)
costs = dts.query_costs_device(idx, Q1, 0.02, block=64)
torch.cuda.synchronize()
print("sanitize workload 2 ok", r2.shape[0], res1.count, int(costs.sum()), flush=True)
# spill path (output-heavy tiles), re-run path is exercised by DTS_SPILL_CAP in the tests
c2 = synth.make_config("C2", scale=0.004)
idx = dts.build_index(c2.D)
r3 = dts.search(idx, c2.Q, 8.0)
idx.free()
print("sanitize workload 3 ok", r3.shape[0], flush=True)
# long-segment outliers: copies, canonical filter in staged tiles, spilled
# records filtered after pass 1 (k_spill_filter), count-only filter
g = np.random.default_rng(17)
n = 3000
D = np.zeros((n, 8))
D[:, 4] = 1.0
D[:, 1:4] = g.uniform(0, 0.05, (n, 3))
D[:, 5:8] = D[:, 1:4] + g.uniform(-0.002, 0.002, (n, 3))
L = np.zeros((24, 8))
L[:, 4] = 1.0
L[:, 1], L[:, 5] = -15.0, 15.0
L[:, [2, 3]] = g.uniform(0, 0.05, (24, 2))
L[:, [6, 7]] = L[:, [2, 3]]
D = np.ascontiguousarray(np.concatenate([D, L]))
Q = np.ascontiguousarray(D[g.choice(n, 300, replace=False)])
idx = dts.build_index(D)
assert idx.info()["outlier_rows"] >= 20
r4 = dts.search(idx, Q, 0.01)
tot4 = dts.search_count(idx, Q, 0.01)[0]
idx.free()
# temporal shards in host memory (mem_budget_bytes), streamed results
c5 = synth.make_config("C2", scale=0.01)
idx = dts.build_index(c5.D, mem_budget_bytes=70 << 20)
assert idx.info()["shards"] >= 2
r5 = dts.search(idx, c5.Q, 2.0)
chunks = []
dts.search_stream(idx, c5.Q, 2.0, lambda a: chunks.append(a.shape[0]), chunk_results=5000)
idx.free()
print("sanitize workload 4 ok", r4.shape[0], tot4, r5.shape[0], sum(chunks), flush=True)
