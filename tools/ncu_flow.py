"""Per-instruction stall samples of one kernel in program order (phase view)."""
import csv
import io
import subprocess
import sys

rep, kern = sys.argv[1], sys.argv[2]
minpct = float(sys.argv[3]) if len(sys.argv) > 3 else 0.5
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass", "-k", kern, "-c", "1"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hi = [i for i, x in enumerate(rows) if 'Source' in x and 'Address' in x][0]
h = rows[hi]
si, wi = h.index('Source'), h.index('Warp Stall Sampling (All Samples)')
st = [(i, c) for i, c in enumerate(h) if c.startswith('stall_') and 'Not Issued' not in c]
data = []
seen = set()
for x in rows[hi + 1:]:
    if len(x) <= wi or not x[wi].isdigit() or x[0] in seen:
        continue
    seen.add(x[0])
    data.append(x)
tot = sum(int(x[wi]) for x in data) or 1
print("samples", tot)
acc = 0
for x in data:
    a = int(x[wi])
    acc += a
    if 100 * a / tot >= minpct:
        reasons = sorted(((int(x[i] or 0), c[6:]) for i, c in st), reverse=True)[:2]
        rs = " ".join(f"{c}={v}" for v, c in reasons if v)
        print(f"{100 * a / tot:5.1f}% cum={100 * acc / tot:5.1f}% {x[si].strip()[:60]:60s} {rs}")
