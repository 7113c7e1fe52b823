"""Median per-kernel metrics from an ncu --csv metrics run (python tools/kprof_summary.py file.csv)."""
import collections
import csv
import sys

rows = [r for r in csv.reader(open(sys.argv[1])) if len(r) > 10]
h = rows[0]
ki, mi, vi = h.index("Kernel Name"), h.index("Metric Name"), h.index("Metric Value")
agg = collections.defaultdict(lambda: collections.defaultdict(list))
for r in rows[1:]:
    k = r[ki].split("(")[0].replace("void ", "").split("::")[-1]
    agg[k][r[mi]].append(float(r[vi].replace(",", "")))
for k, d in agg.items():
    print(k, {m: round(sorted(v)[len(v) // 2], 2) for m, v in d.items()}, "n =", len(d["gpu__time_duration.sum"]))
