"""Markdown table of a sweep JSONL (scripts/sweep.py), with the paper's own
response times beside the paper-replica scenarios (context only: Tesla C2075,
OpenCL, different data instances)."""
import json
import sys

PAPER = {  # (config, method, d) -> (seconds, what), BASELINE.md / P:L154-P:L169
    ("S1", "temporal", 50.0): (1.21, "GPUTemporal, C2075 (P:L154)"),
    ("S1", "subbin", 50.0): (1.36, "GPUSpatioTemporal v=1, C2075 (P:L154)"),
    ("S2", "subbin", 0.001): (41.75, "GPUSpatioTemporal, C2075 (P:L162); CPU-RTree 9.70 s"),
    ("S2", "subbin", 5.0): (116.09, "GPUSpatioTemporal, C2075 (P:L162); CPU-RTree 184.4 s"),
}

rows = [json.loads(l) for l in open(sys.argv[1]) if l.strip() and not l.startswith("#")]
print("| config | method | d | results | candidates | device search ms | response time ms "
      "(host Q -> host results) | q-seg/s (response) | paper (context) |")
print("|---|---|---|---|---|---|---|---|---|")
for r in rows:
    p = PAPER.get((r["config"], r["method"], float(r["d"])))
    ptxt = f"{p[0]} s — {p[1]}" if p else ""
    dev = f"{r['search_ms_device']:.3f}" if r["search_ms_device"] else "streamed"
    cand = f"{r['candidates']:,}" if r["candidates"] is not None else "—"
    print(f"| {r['config']} | {r['method']} | {r['d']} | {r['results']:,} | {cand} | {dev} | "
          f"{1e3 * r['response_time_s']:.2f} | {r['qseg_per_s_response']:.3g} | {ptxt} |")
