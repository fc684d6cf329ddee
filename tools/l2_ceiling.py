"""Parse tools/gather_bench.cu output into profiles/r03/l2_ceiling.json: the
highest random 4-byte request rate (ld.cg gathers or red.min reductions on a
C2-sized label array) over the launch shapes tried.
Usage: python tools/l2_ceiling.py gather_bench.txt > profiles/r03/l2_ceiling.json"""
import json
import re
import sys

lines = open(sys.argv[1]).read().splitlines()
rows = []
for ln in lines:
    m = re.match(r"(\S+)\s+R=\s*(\d+) blocks/SM=\s*(\d+) threads=\s*(\d+) : +([\d.]+) G accesses/s", ln)
    if m:
        rows.append({"op": m.group(1), "R": int(m.group(2)), "blocks_per_sm": int(m.group(3)),
                     "threads": int(m.group(4)), "g_per_s": float(m.group(5))})
best = max((r for r in rows if r["op"] in ("ld.cg", "redMin")), key=lambda r: r["g_per_s"])
print(json.dumps({"ceiling_g_per_s": best["g_per_s"], "best": best, "rows": rows,
                  "source": "tools/gather_bench.cu: random 4-byte ld.cg / red.min on a 16.8 MB (C2) label array, "
                            "max over launch shapes, one B200"}, indent=1))
