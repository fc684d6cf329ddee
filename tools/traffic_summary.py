"""dram traffic vs algorithmic bytes of the SAME expand launches.

Inputs: an ncu CSV (--metrics gpu__time_duration.sum,dram__bytes_read.sum,
dram__bytes_write.sum, -k regex:expand_warp) of `tools/prof_run.py --json S`
in host-loop mode, and S (per-call statistics of those very launches).
Algorithmic bytes: BFS 8 B per relaxed edge + 20 B per active
vertex, SSSP 12 + 24, CC 8 + 24.  Output: JSON on stdout.
Usage: python tools/traffic_summary.py launches.csv stats.json"""
import csv
import json
import sys

BPE = {"bfs": 8, "sssp": 12, "cc": 8, "sswp": 12}
BPV = {"bfs": 20, "sssp": 24, "cc": 24, "sswp": 24}
rows = list(csv.reader(open(sys.argv[1])))
hdr = next(r for r in rows if r and r[0] == "ID")
per = {}
for r in rows:
    if len(r) != len(hdr) or r[0] == "ID":
        continue
    d = dict(zip(hdr, r))
    if "expand" not in d["Kernel Name"]:
        continue
    v = float(d["Metric Value"].replace(",", ""))
    u = d["Metric Unit"].lower()
    scale = {"byte": 1, "kbyte": 1e3, "mbyte": 1e6, "gbyte": 1e9, "nsecond": 1e-3, "ns": 1e-3, "usecond": 1, "us": 1, "msecond": 1e3, "ms": 1e3}
    per.setdefault(d["ID"], {})[d["Metric Name"]] = v * scale.get(u, 1)
stats = json.load(open(sys.argv[2]))
alg_bytes = sum(BPE[c["alg"]] * c["edges_processed"] + BPV[c["alg"]] * c["frontier_total"] for c in stats["calls"])
L = len(per)
dram = sum(x.get("dram__bytes_read.sum", 0) + x.get("dram__bytes_write.sum", 0) for x in per.values())
us = sum(x.get("gpu__time_duration.sum", 0) for x in per.values())
out = {"config": stats["config"], "algs": sorted({c["alg"] for c in stats["calls"]}), "launches": L,
       "alg_bytes_total": alg_bytes, "dram_bytes_total": dram,
       "alg_bytes_per_launch": alg_bytes / max(L, 1), "dram_bytes_per_launch": dram / max(L, 1),
       "dram_over_alg": dram / max(alg_bytes, 1), "ncu_expand_us_total": us,
       "alg_gbs_under_ncu": alg_bytes / max(us, 1e-9) / 1e3, "dram_gbs_under_ncu": dram / max(us, 1e-9) / 1e3,
       "how": "ncu --cache-control none --clock-control none over every expand launch of one host-loop call per "
              "algorithm (tools/prof_run.py); algorithmic bytes from the same calls' etg_stats"}
# L2 requests / sectors from the SM side (when the capture has them): the
# expand's real bound on L2-resident configs is the random-request rate
req = sum(x.get("lts__t_requests_srcunit_tex.sum", 0) for x in per.values())
sec = sum(x.get("lts__t_sectors_srcunit_tex.sum", 0) for x in per.values())
if req:
    edges = sum(c["edges_processed"] for c in stats["calls"])
    out.update({"l2_requests_total": req, "l2_sectors_total": sec,
                "l2_requests_per_launch": req / max(L, 1), "l2_sectors_per_launch": sec / max(L, 1),
                "l2_requests_per_edge": req / max(edges, 1),
                "l2_g_requests_per_s_under_ncu": req / max(us, 1e-9) / 1e3})
print(json.dumps(out, indent=1))
