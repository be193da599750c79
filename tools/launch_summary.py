"""Summarise an ncu launch list (--metrics gpu__time_duration.sum,dram__bytes_read.sum,
dram__bytes_write.sum --csv) of the bench command into a markdown table for profiles/."""
import collections
import csv
import sys

path = sys.argv[1]
rows = [r for r in csv.reader(open(path)) if len(r) > 10]
h = rows[0]
ki, mi, vi, ii = h.index("Kernel Name"), h.index("Metric Name"), h.index("Metric Value"), h.index("ID")
per = collections.defaultdict(dict)
names = {}
for r in rows[1:]:
    per[int(r[ii])][r[mi]] = float(r[vi].replace(",", ""))
    names[int(r[ii])] = r[ki]
agg = collections.defaultdict(lambda: [0, 0.0, 0.0])
for i, m in per.items():
    n = names[i].split("(")[0].replace("void ", "").replace("aabft::<unnamed>::", "")
    a = agg[n]
    a[0] += 1
    a[1] += m.get("gpu__time_duration.sum", 0.0)
    a[2] += m.get("dram__bytes_read.sum", 0.0) + m.get("dram__bytes_write.sum", 0.0)
unit = "ns"
print("| kernel | launches | us/launch | DRAM MB/launch | DRAM GB/s |")
print("|---|---|---|---|---|")
for n, (c, t, b) in sorted(agg.items(), key=lambda x: -x[1][1]):
    us = t / c / 1e3
    print(f"| `{n[:90]}` | {c} | {us:.1f} | {b / c / 1e6:.1f} | {b / t if t else 0:.0f} |")
