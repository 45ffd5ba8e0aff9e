"""Per-source-line executed warp instructions of one kernel in an .ncu-rep
(ncu --page source --print-source cuda,sass), top lines first."""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 30
units = float(sys.argv[3]) if len(sys.argv) > 3 else 0.0
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
fname, hdr, agg, total = "?", None, [], 0.0
for r in rows:
    if not r:
        continue
    if r[0] == "File Path":
        fname = r[1].split("/")[-1]
        continue
    if r[0] == "Line No":
        hdr = r
        continue
    if hdr is None or len(r) != len(hdr) or r[2] != "-":
        continue
    try:
        v = float(r[hdr.index("Instructions Executed")] or 0)
    except ValueError:
        continue
    if v > 0:
        agg.append((v, f"{fname}:{r[0]}", r[1].strip()[:80]))
        total += v
agg.sort(reverse=True)
print(f"total warp instructions {total:.4g}" + (f", per unit {total / units:.1f}" if units else ""))
for v, loc, src in agg[:top]:
    print(f"{100 * v / total:5.1f}% {loc:18s} {src}")
