"""Aggregate an ncu --metrics CSV over the launches of one kernel family:
sums for counters (bytes, sectors, requests, instructions, time), time-weighted
means for percentages.  Usage: python tools/ncu_agg.py file.csv [kernel-substring]"""
import csv
import json
import sys

rows = list(csv.reader(open(sys.argv[1])))
key = sys.argv[2] if len(sys.argv) > 2 else "expand"
hdr = next(r for r in rows if r and r[0] == "ID")
per = {}
scale = {"byte": 1, "kbyte": 1e3, "mbyte": 1e6, "gbyte": 1e9, "nsecond": 1e-3, "ns": 1e-3, "usecond": 1, "us": 1, "msecond": 1e3, "ms": 1e3}
for r in rows:
    if len(r) != len(hdr) or r[0] == "ID":
        continue
    d = dict(zip(hdr, r))
    if key not in d["Kernel Name"]:
        continue
    try:
        v = float(d["Metric Value"].replace(",", ""))
    except ValueError:
        continue
    per.setdefault(d["ID"], {})[d["Metric Name"]] = v * scale.get(d["Metric Unit"].lower(), 1)
t = {i: x.get("gpu__time_duration.sum", 0.0) for i, x in per.items()}
T = sum(t.values()) or 1.0
names = sorted({m for x in per.values() for m in x})
out = {"launches": len(per), "time_us": T}
for m in names:
    if m == "gpu__time_duration.sum":
        continue
    if m.endswith(".pct") or "pct_of_peak" in m:
        out[m + " (time-weighted)"] = sum(x.get(m, 0) * t[i] for i, x in per.items()) / T
    else:
        out[m] = sum(x.get(m, 0) for x in per.values())
print(json.dumps(out, indent=1))
