"""Top SASS lines by warp-stall samples for one kernel of an ncu report."""
import csv
import io
import subprocess
import sys

rep, kern = sys.argv[1], sys.argv[2]
top = int(sys.argv[3]) if len(sys.argv) > 3 else 25
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass", "-k", kern, "-c", "1"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hi = [i for i, x in enumerate(rows) if 'Source' in x and 'Address' in x][0]
h = rows[hi]
si, wi, ei = h.index('Source'), h.index('Warp Stall Sampling (All Samples)'), h.index('Instructions Executed')
data = [(int(x[wi]), x[si].strip(), x[ei]) for x in rows[hi + 1:] if len(x) > wi and x[wi].isdigit()]
tot = sum(a for a, _, _ in data) or 1
print("samples", tot)
for a, s, e in sorted(data, reverse=True)[:top]:
    print(f"{a:6d} {100 * a / tot:5.1f}% exec={e:>8s} {s[:90]}")
