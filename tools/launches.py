"""Summarise an ncu --metrics gpu__time_duration.sum CSV launch list."""
import collections
import csv
import sys

rows = [r for r in csv.reader(open(sys.argv[1])) if len(r) > 10]
h = rows[0]
ik, iv = h.index('Kernel Name'), h.index('Metric Value')
agg = collections.defaultdict(list)
for r in rows[1:]:
    try:
        agg[r[ik][:48]].append(float(r[iv]))
    except ValueError:
        pass
tot = sum(sum(v) for v in agg.values())
for k, v in sorted(agg.items(), key=lambda kv: -sum(kv[1])):
    print(f"{k:50s} n={len(v):5d} mean={sum(v)/len(v)/1e3:9.1f} us total={sum(v)/1e6:8.2f} ms  {100*sum(v)/tot:5.1f}%")
