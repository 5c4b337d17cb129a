"""Summarise an ncu --metrics gpu__time_duration.sum CSV launch list: per-kernel count / mean / total."""
import collections
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
hi = next(i for i, r in enumerate(rows) if 'Kernel Name' in r)
h = rows[hi]
ki, vi, ui = h.index('Kernel Name'), h.index('Metric Value'), h.index('Metric Unit')
agg = collections.defaultdict(list)
for r in rows[hi + 1:]:
    if len(r) <= vi:
        continue
    name = r[ki].split('(')[0].split('::')[-1]
    v = float(r[vi].replace(',', ''))
    v = {'ns': v / 1000, 'nsecond': v / 1000, 'us': v, 'usecond': v, 'ms': v * 1000, 'msecond': v * 1000}[r[ui]]
    agg[name].append(v)
skip = int(sys.argv[2]) if len(sys.argv) > 2 else 0
tot = sum(sum(v[skip:]) for v in agg.values())
for k, v in sorted(agg.items(), key=lambda x: -sum(x[1][skip:])):
    vv = v[skip:] or v
    print(f"{k:32s} n={len(v):4d} mean={sum(vv)/len(vv):8.2f}us share={100*sum(v[skip:])/tot:5.1f}%")
