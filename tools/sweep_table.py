"""Markdown rows of the per-config sweep (gpurun_out/ev_*.json -> profiles/README.md)."""
import glob
import json
import os
import sys

src = sys.argv[1] if len(sys.argv) > 1 else "gpurun_out"
rows = {}
for p in sorted(glob.glob(os.path.join(src, "ev_*.json"))):
    d = json.load(open(p))
    name = os.path.basename(p)[3:-5]
    rows[name] = d
with open(os.path.join(src, "summary.txt"), "w") as f:
    for name, d in rows.items():
        pa = d["per_alg"]
        f.write(f"{name} {d['value']:.2f} " + str({k: (round(v['gteps'], 1), round(v['ms_per_call'], 3)) for k, v in pa.items()}) + "\n")


def cell(d, a):
    v = d["per_alg"].get(a)
    return f"{v['gteps']:.1f}" if v else ""


for name, d in rows.items():
    print(f"| {name} | {cell(d, 'bfs')} | {cell(d, 'sssp')} | {cell(d, 'cc')} | {d['value']:.1f} |")
