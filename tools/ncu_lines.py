"""Per-source-line totals of an ncu report (warp-stall samples, instructions
executed), from the cuda,sass correlated source page.
Usage: python tools/ncu_lines.py rep.ncu-rep [N]"""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
N = int(sys.argv[2]) if len(sys.argv) > 2 else 25
txt = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(txt)))
hdr = next(r for r in rows if r and r[0] == "Line No")
ismp = hdr.index("Warp Stall Sampling (All Samples)")
iins = hdr.index("Instructions Executed")
agg = {}
tot_s = tot_i = 0
for r in rows:
    if len(r) != len(hdr) or r[0] in ("Line No", ""):
        continue
    try:
        s, i = int(r[ismp] or 0), int(r[iins] or 0)
    except ValueError:
        continue
    key = (int(r[0]), r[1].strip()[:90])
    a = agg.setdefault(key, [0, 0])
    a[0] += s
    a[1] += i
    tot_s += s
    tot_i += i
print(f"samples {tot_s}, warp instructions {tot_i}")
for (ln, src), (s, i) in sorted(agg.items(), key=lambda x: -x[1][0])[:N]:
    print(f"{100 * s / max(tot_s, 1):5.1f}% smp {100 * i / max(tot_i, 1):5.1f}% ins  L{ln:5d} {src}")
