"""The paper's largest-output point: S2 (25,165,824 entries, 50,880 queries,
P:L140) at d = 5 (116.09 s on the paper's GPU), 7.5e9 results.
Count-only search (dts_search_count) and the full streamed search
(dts_search_stream: every result copied to the host in canonical chunks; the
callback folds a checksum) -- the paper's incremental processing of Q when
the result set exceeds memory.  Index build excluded.
One JSON line."""
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ipps_gowanlockc15_b200 as dts  # noqa: E402
import synth  # noqa: E402

d = float(sys.argv[1]) if len(sys.argv) > 1 else 5.0
c = synth.make_config("S2")
t0 = time.perf_counter()
idx = dts.build_index(c.D, d_hint=d)
torch.cuda.synchronize()
t_build = time.perf_counter() - t0
dts.search_count(idx, c.Q[:512], d)                       # warm-up
t0 = time.perf_counter()
total, counts, cst = dts.search_count(idx, c.Q, d, time_kernels=True)
t_count = time.perf_counter() - t0
state = {"n": 0, "chunks": 0, "x": 0, "last": -1}


def fold(ch):
    # cheap per-chunk checks: canonical order across chunk boundaries (first
    # and last keys), a sum of the entry ids as a checksum
    state["n"] += ch.shape[0]
    state["chunks"] += 1
    k0 = (int(ch["query_id"][0]) << 32) | int(ch["entry_id"][0])
    k1 = (int(ch["query_id"][-1]) << 32) | int(ch["entry_id"][-1])
    assert k0 > state["last"] and k1 >= k0
    state["last"] = k1
    state["x"] += int(ch["entry_id"].sum(dtype=np.uint64))


t0 = time.perf_counter()
st = dts.search_stream(idx, c.Q, d, fold)
t_stream = time.perf_counter() - t0
# the library's own cost: every result delivered, the callback only counts
nres = {"n": 0}


def count_only(ch):
    nres["n"] += ch.shape[0]


t0 = time.perf_counter()
dts.search_stream(idx, c.Q, d, count_only)
t_stream_lib = time.perf_counter() - t0
assert nres["n"] == state["n"]
print(json.dumps({"config": "S2", "d": d, "n_entries": int(c.D.shape[0]),
                  "n_queries": int(c.Q.shape[0]), "results": total,
                  "results_streamed": state["n"], "chunks": state["chunks"],
                  "max_per_query": int(counts.max()), "count_s": t_count,
                  "count_pass_ms": cst["ms_count"], "candidates": cst["candidates"],
                  "stream_s": t_stream, "stream_count_cb_s": t_stream_lib, "build_s": t_build,
                  "paper_s": 116.09 if d == 5.0 else None,
                  "note": "count_s: dts_search_count (host Q -> per-query counts); stream_s: "
                          "dts_search_stream, every result in canonical order to the host "
                          "(pinned chunks, checksum callback; stream_count_cb_s: the callback only counts); paper: GPUSpatioTemporal on its "
                          "GPU, P:L162 (context only)"}), flush=True)
