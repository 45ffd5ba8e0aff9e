"""Summarise an ncu launch-list CSV (gpu__time_duration per launch): per-kernel
totals of the last search call (from its query-key kernel on), or of the
last `frac` of the launches when the list has no search."""
import collections
import csv
import sys

path = sys.argv[1]
frac = float(sys.argv[2]) if len(sys.argv) > 2 else 0.5
rows = list(csv.reader(open(path)))
hdr = None
data = []
for r in rows:
    if r and r[0] == "ID":
        hdr = r
        continue
    if hdr and len(r) == len(hdr):
        data.append(dict(zip(hdr, r)))
agg = collections.OrderedDict()
start = int(len(data) * (1 - frac))
qk = [i for i, r in enumerate(data) if "k_qkeys" in r["Kernel Name"]]
if qk:
    start = qk[-1]
for r in data[start:]:
    name = r["Kernel Name"].split("(")[0].replace("(anonymous namespace)::", "")[:48]
    v = float(r["Metric Value"])
    agg.setdefault(name, [0.0, 0])
    agg[name][0] += v
    agg[name][1] += 1
tot = sum(v[0] for v in agg.values())
for k, v in sorted(agg.items(), key=lambda x: -x[1][0]):
    print(f"{v[0] / 1e3:9.1f} us {v[1]:3d}x {100 * v[0] / tot:5.1f}%  {k}")
print(f"total {tot / 1e3:.1f} us over {len(data) - start} launches (unit {data[-1]['Metric Unit']})")
