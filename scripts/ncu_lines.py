"""Per-source-line warp-stall samples of one kernel in an .ncu-rep
(ncu --page source --print-source cuda,sass), top lines first."""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 25
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
fname = "?"
hdr = None
agg = []
total = 0
for r in rows:
    if not r:
        continue
    if r[0] == "File Path":
        fname = r[1].split("/")[-1]
        continue
    if r[0] == "Line No":
        hdr = r
        continue
    if hdr is None or r[0] in ("Function Name",) or len(r) != len(hdr):
        continue
    if r[2] != "-":          # sass rows carry an address; cuda rows have '-'
        continue
    try:
        s = int(r[hdr.index("Warp Stall Sampling (All Samples)")])
    except ValueError:
        continue
    cols = {k: r[i] for i, k in enumerate(hdr) if k.startswith("stall_") and "Not Issued" not in k}
    top3 = sorted(((int(v) if v.isdigit() else 0, k[6:]) for k, v in cols.items()), reverse=True)[:3]
    agg.append((s, f"{fname}:{r[0]}", r[1].strip()[:70], top3))
    total += s
agg.sort(reverse=True)
print(f"total samples {total}")
for s, loc, src, t3 in agg[:top]:
    print(f"{100 * s / max(total, 1):5.1f}% {loc:18s} {src:70s} {' '.join(f'{k}={v}' for v, k in t3)}")
