"""profiles/traffic.json from a single-pass steady-state ncu metric list of the
default bench command (tools/checkpoint.sh): per kernel, the mean DRAM bytes
(read + write) per launch -- the roofline line's "traffic" -- and the commit the
capture was taken from.  usage: python tools/traffic_json.py launches.csv <tag> <git-sha>"""
import collections
import csv
import json
import sys

path, tag, sha = sys.argv[1], sys.argv[2], sys.argv[3]
rows = list(csv.reader(open(path)))
hi = next(i for i, r in enumerate(rows) if 'Kernel Name' in r)
h = rows[hi]
ki, ii, mi, vi, ui = (h.index('Kernel Name'), h.index('ID'), h.index('Metric Name'), h.index('Metric Value'),
                      h.index('Metric Unit'))
scale = {'ns': 1e-3, 'nsecond': 1e-3, 'us': 1, 'usecond': 1, 'ms': 1e3, 'msecond': 1e3, 'byte': 1,
         'Kbyte': 1e3, 'Mbyte': 1e6, 'Gbyte': 1e9}
per = collections.defaultdict(dict)
names = {}
for r in rows[hi + 1:]:
    if len(r) > vi:
        names[r[ii]] = r[ki].split('(')[0].split('::')[-1]
        per[r[ii]][r[mi]] = float(r[vi].replace(',', '')) * scale.get(r[ui], 1)
agg = collections.defaultdict(list)
for i in sorted(per, key=int):
    agg[names[i]].append(per[i])
out = {}
for k, v in agg.items():
    v = v[3:] or v   # (the first launches are warm-up batches)
    out[k] = {"dram_bytes_per_launch": sum(m.get('dram__bytes_read.sum', 0) + m.get('dram__bytes_write.sum', 0)
                                           for m in v) / len(v),
              "us_per_launch": sum(m.get('gpu__time_duration.sum', 0) for m in v) / len(v),
              "launches": len(v),
              "source": f"ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum "
                        f"--cache-control none --clock-control none (single pass, no replay: steady-state "
                        f"caches), bench cfg2 --steps 8 --warmup 3, checkpoint {tag}, commit {sha}"}
json.dump(out, open("profiles/traffic.json", "w"), indent=1)
print(json.dumps({k: round(v["dram_bytes_per_launch"] / 1e6, 2) for k, v in out.items()}))
