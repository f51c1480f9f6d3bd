"""Summarise an ncu launch list (--metrics gpu__time_duration.sum --csv) per kernel."""
import collections
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
start = next(i for i, r in enumerate(rows) if r and r[0] == "ID")
hdr = rows[start]
iN, iV, iM = hdr.index("Kernel Name"), hdr.index("Metric Value"), hdr.index("Metric Name")
agg = collections.defaultdict(lambda: [0, 0.0])
for r in rows[start + 1:]:
    if len(r) <= iV or r[iM] != "gpu__time_duration.sum":
        continue
    name = r[iN].split("(")[0].replace("void ", "")
    agg[name][0] += 1
    agg[name][1] += float(r[iV].replace(",", ""))
tot = sum(v[1] for v in agg.values())
print(f"{'kernel':32s} {'launches':>8s} {'total_ms':>10s} {'avg_us':>10s} {'share':>6s}")
for k, v in sorted(agg.items(), key=lambda kv: -kv[1][1]):
    print(f"{k:32s} {v[0]:8d} {v[1] / 1e6:10.3f} {v[1] / v[0] / 1e3:10.2f} {v[1] / tot:6.3f}")
print(f"{'TOTAL':32s} {sum(v[0] for v in agg.values()):8d} {tot / 1e6:10.3f}")
