"""Top CUDA source lines by warp-stall samples for one kernel of an ncu report (-lineinfo build):
    python tools/ncu_lines.py REPORT KERNEL [TOP] [LAUNCH_INDEX]"""
import csv
import io
import os
import subprocess
import sys

rep, kern = sys.argv[1], sys.argv[2]
top = int(sys.argv[3]) if len(sys.argv) > 3 else 30
skip = sys.argv[4] if len(sys.argv) > 4 else "0"
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass", "-k", kern,
                      "-s", skip, "-c", "1"], capture_output=True, text=True).stdout
f = "?"
data = []
hdr = None
for x in csv.reader(io.StringIO(out)):
    if len(x) == 2 and x[0] == "File Path":
        f = os.path.basename(x[1])
        continue
    if x and x[0] == "Line No":
        hdr = x
        continue
    if hdr is None or len(x) < 8 or not x[0] or x[2] != "-":
        continue
    si = hdr.index("Warp Stall Sampling (All Samples)")
    ei = hdr.index("Instructions Executed")
    if x[si].isdigit():
        st = sorted(((float(x[j] or 0), hdr[j][6:]) for j in range(len(hdr))
                     if hdr[j].startswith("stall_") and "Not Issued" not in hdr[j] and x[j] not in ("", "-")),
                    reverse=True)
        xs = hdr.index("L1 Wavefronts Shared Excessive") if "L1 Wavefronts Shared Excessive" in hdr else None
        exc = x[xs] if xs is not None else ""
        why = " ".join(f"{n}:{int(v)}" for v, n in st[:3] if v > 0)
        data.append((int(x[si]), f"{f}:{x[0]}", x[ei], x[1].strip(), why, exc))
tot = sum(d[0] for d in data) or 1
print("samples", tot)
for a, loc, e, s, why, exc in sorted(data, reverse=True)[:top]:
    print(f"{a:6d} {100 * a / tot:5.1f}% {loc:24s} exec={e:>9s} [{why}] smem_excess={exc} | {s[:70]}")
