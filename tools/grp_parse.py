"""Summarise EIRENE_GROUP_PROF lines (groups slower than 20 us): counts per
mode and the slowest groups per phase (diagnostic)."""
import collections
import re
import sys

rows = []
for line in open(sys.argv[1]):
    m = re.search(r"ticket (\d+) cnt (\d+) mode (\d+) sort ([\d.]+) sweep1 ([\d.]+) lookback ([\d.]+) emit ([\d.]+)", line)
    if m:
        rows.append(tuple(float(x) for x in m.groups()))
print("slow groups", len(rows), "modes", dict(collections.Counter(int(r[2]) for r in rows)))
for key, name in [(3, "sort"), (4, "sweep1"), (5, "lookback"), (6, "emit")]:
    top = sorted(rows, key=lambda r: -r[key])[:3]
    print(f"{name:8s}", [(int(r[1]), int(r[2]), r[key]) for r in top])
