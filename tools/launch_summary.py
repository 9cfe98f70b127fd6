"""Summarise an ncu --csv launch list (gpu__time_duration.sum): per kernel count, total and
first/last durations (development aid).  Usage: python tools/launch_summary.py file.csv"""
import collections
import csv
import sys

lines = [l for l in open(sys.argv[1]) if l.startswith('"')]
rows = list(csv.DictReader(lines))
agg = collections.defaultdict(list)
order = []
for r in rows:
    if r["Metric Name"] != "gpu__time_duration.sum":
        continue
    k = r["Kernel Name"].split("(")[0]
    if k not in agg:
        order.append(k)
    agg[k].append(float(r["Metric Value"]) / 1e3)
tot = sum(sum(v) for v in agg.values())
print(f"{len(rows)} launches, {tot:.1f} us serialised")
for k in order:
    v = agg[k]
    print(f"{k[:60]:60s} n={len(v):4d} total {sum(v):9.1f} us ({100*sum(v)/tot:4.1f}%)  first {[round(x,1) for x in v[:4]]} last {[round(x,1) for x in v[-3:]]}")
