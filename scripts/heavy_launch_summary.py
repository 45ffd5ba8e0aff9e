"""Per-kernel device time of the last search call in ncu launch-list CSVs
(scripts/heavy_launches.sh)."""
import collections
import csv
import sys

for f in sys.argv[1:]:
    rows = [r for r in csv.reader(open(f)) if r]
    hdr = next(r for r in rows if r[0] == "ID")
    data = [r for r in rows if r[0].isdigit()]
    ik, iv = hdr.index("Kernel Name"), hdr.index("Metric Value")
    last = max(i for i, r in enumerate(data) if "k_qkeys" in r[ik])
    agg = collections.OrderedDict()
    for r in data[last:]:
        k = r[ik][:70]
        agg.setdefault(k, [0.0, 0])
        agg[k][0] += float(r[iv].replace(",", ""))
        agg[k][1] += 1
    tot = sum(v[0] for v in agg.values())
    print(f, "total %.3f ms" % (tot / 1e6))
    for k, v in sorted(agg.items(), key=lambda x: -x[1][0])[:16]:
        print("  %9.3f ms %4dx  %s" % (v[0] / 1e6, v[1], k))
