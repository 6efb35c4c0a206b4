"""Summarise an `ncu --metrics gpu__time_duration.sum --csv` launch list: the library's
kernels (pfpl::*) with launch count, mean and total time and share of library time.
usage: launches_md.py LAUNCHES.csv"""
import csv
import sys
from collections import defaultdict

lines = [l for l in open(sys.argv[1]) if l.startswith('"')]
rows = list(csv.reader(lines))
h = rows[0]
ik, im, iv = h.index("Kernel Name"), h.index("Metric Name"), h.index("Metric Value")
agg = defaultdict(list)
for r in rows[1:]:
    if r[im] != "gpu__time_duration.sum" or "pfpl::" not in r[ik]:
        continue
    name = r[ik].split("(")[0]
    agg[name].append(float(r[iv].replace(",", "")) / 1000.0)
tot = sum(sum(v) for v in agg.values())
print("| kernel | launches | mean us | max us | total us | share of library time |")
print("|---|---|---|---|---|---|")
for k, v in sorted(agg.items(), key=lambda kv: -sum(kv[1])):
    print(f"| `{k}` | {len(v)} | {sum(v) / len(v):.1f} | {max(v):.1f} | {sum(v):.1f} | {100 * sum(v) / tot:.1f}% |")
