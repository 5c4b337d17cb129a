"""Per-kernel mean duration and DRAM bytes per launch from a SINGLE-PASS ncu
metric list (--metrics gpu__time_duration.sum,dram__bytes_read.sum,
dram__bytes_write.sum --cache-control none --clock-control none --csv): no
kernel replay, caches not flushed, so the bytes are the steady-state traffic of
the timed run (unlike a --set full capture, whose replays restore memory).
usage: python tools/traffic1.py launches.csv [skip_first_n_per_kernel]"""
import collections
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
hi = next(i for i, r in enumerate(rows) if 'Kernel Name' in r)
h = rows[hi]
ki, ii, mi, vi, ui = (h.index('Kernel Name'), h.index('ID'), h.index('Metric Name'), h.index('Metric Value'),
                      h.index('Metric Unit'))
scale = {'ns': 1e-3, 'nsecond': 1e-3, 'us': 1, 'usecond': 1, 'ms': 1e3, 'msecond': 1e3,
         'byte': 1, 'Kbyte': 1e3, 'Mbyte': 1e6, 'Gbyte': 1e9, 'KB': 1e3, 'MB': 1e6, 'GB': 1e9}
per = collections.defaultdict(dict)
names = {}
for r in rows[hi + 1:]:
    if len(r) <= vi:
        continue
    names[r[ii]] = r[ki].split('(')[0].split('::')[-1]
    per[r[ii]][r[mi]] = float(r[vi].replace(',', '')) * scale.get(r[ui], 1)
agg = collections.defaultdict(list)
for i in sorted(per, key=int):
    agg[names[i]].append(per[i])
skip = int(sys.argv[2]) if len(sys.argv) > 2 else 0
tot = sum(sum(m.get('gpu__time_duration.sum', 0) for m in v[skip:]) for v in agg.values()) or 1
for k, v in sorted(agg.items(), key=lambda x: -sum(m.get('gpu__time_duration.sum', 0) for m in x[1][skip:])):
    vv = v[skip:] or v
    d = sum(m.get('gpu__time_duration.sum', 0) for m in vv) / len(vv)
    rd = sum(m.get('dram__bytes_read.sum', 0) for m in vv) / len(vv)
    wr = sum(m.get('dram__bytes_write.sum', 0) for m in vv) / len(vv)
    sh = 100 * sum(m.get('gpu__time_duration.sum', 0) for m in v[skip:]) / tot
    print(f"{k:28s} n={len(v):4d} dur={d:8.2f}us share={sh:5.1f}% dramR={rd / 1e6:8.2f}MB dramW={wr / 1e6:7.2f}MB "
          f"dram_GBps={(rd + wr) / (d * 1e3) if d else 0:7.1f}")
