"""Hottest SASS instructions of an ncu report (warp-stall samples), with the
CUDA source line each maps to.  Usage: python tools/ncu_hot.py rep.ncu-rep [N]"""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
N = int(sys.argv[2]) if len(sys.argv) > 2 else 25
sass = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                      capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(sass)))
hdr = rows[1]
ia, isrc, ismp = hdr.index("Address"), hdr.index("Source"), hdr.index("Warp Stall Sampling (All Samples)")
recs = []
for r in rows[2:]:
    if len(r) != len(hdr):
        continue
    try:
        recs.append((int(r[ismp] or 0), r[ia], r[isrc]))
    except ValueError:
        pass
tot = sum(x[0] for x in recs) or 1
print(f"total samples {tot}")
for smp, a, src in sorted(recs, reverse=True)[:N]:
    print(f"{smp:7d} {100 * smp / tot:5.1f}%  {a}  {src[:110]}")
