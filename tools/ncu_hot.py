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
stalls = [(i, h[6:]) for i, h in enumerate(hdr) if h.startswith("stall_") and "Not Issued" not in h]
recs = []
tot_by = {}
for r in rows[2:]:
    if len(r) != len(hdr):
        continue
    try:
        by = sorted(((int(r[i] or 0), nm) for i, nm in stalls), reverse=True)
        for v, nm in by:
            tot_by[nm] = tot_by.get(nm, 0) + v
        recs.append((int(r[ismp] or 0), r[ia], r[isrc], by[:2]))
    except ValueError:
        pass
tot = sum(x[0] for x in recs) or 1
print(f"total samples {tot}; by reason:",
      ", ".join(f"{k} {100 * v / tot:.1f}%" for k, v in sorted(tot_by.items(), key=lambda x: -x[1])[:8]))
for smp, a, src, by in sorted(recs, reverse=True)[:N]:
    why = " ".join(f"{nm}:{v}" for v, nm in by if v)
    print(f"{smp:7d} {100 * smp / tot:5.1f}%  {a[-5:]}  {src[:70]:70s} {why}")
