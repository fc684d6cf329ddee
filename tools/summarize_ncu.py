"""Summarise ncu outputs of a round into profiles/ (committed evidence)."""
import csv, io, json, subprocess, sys, collections

def raw(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    r = list(csv.reader(io.StringIO(out)))
    hdr, units = r[0], r[1]
    rows = []
    for vals in r[2:]:
        rows.append({h: (u, v) for h, u, v in zip(hdr, units, vals)})
    return rows

def num(x):
    try: return float(x.replace(",", ""))
    except Exception: return None

KEYS = ["Kernel Name", "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "dram__throughput.avg.pct_of_peak_sustained_elapsed", "lts__t_sector_hit_rate.pct",
        "lts__throughput.avg.pct_of_peak_sustained_elapsed", "l1tex__throughput.avg.pct_of_peak_sustained_active",
        "lts__t_requests_srcunit_tex_op_read.sum", "lts__t_sectors_srcunit_tex_op_atom.sum",
        "lts__t_sectors_srcunit_tex_op_red.sum", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "smsp__inst_executed.sum", "launch__registers_per_thread", "launch__grid_size",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed"]

def summarize_rep(rep):
    rows = raw(rep)
    out = []
    for row in rows:
        d = {}
        for k in KEYS:
            if k in row:
                u, v = row[k]
                d[k] = v if k == "Kernel Name" else num(v)
                if k != "Kernel Name" and u: d[k + " [unit]"] = u
        out.append(d)
    return out

def launches(csvfile):
    rows = list(csv.reader(open(csvfile)))
    hdr = None; seq = []
    for r in rows:
        if r and r[0] == "ID": hdr = r; continue
        if hdr and len(r) == len(hdr):
            d = dict(zip(hdr, r))
            if d["Metric Name"] != "gpu__time_duration.sum": continue
            v = float(d["Metric Value"].replace(",", ""))
            u = d["Metric Unit"]
            v = v / 1000.0 if u in ("ns", "nsecond") else (v * 1000.0 if u in ("ms", "msecond") else v)
            seq.append((d["Kernel Name"].split("(")[0], v))
    agg = collections.defaultdict(lambda: [0, 0.0])
    for n, v in seq: agg[n][0] += 1; agg[n][1] += v
    tot = sum(v for _, v in seq)
    return {"total_us": tot, "kernels": {k: {"launches": c, "us": t, "share": t / tot} for k, (c, t) in
                                         sorted(agg.items(), key=lambda x: -x[1][1])}}

if __name__ == "__main__":
    tag = sys.argv[1]
    res = {"tag": tag,
           "launch_list": launches(f"gpurun_out/launches_{tag}.csv"),
           "bfs_expand_depth3": summarize_rep(f"gpurun_out/ncu_expand_{tag}.ncu-rep"),
           "sssp_expand_depth4": summarize_rep(f"gpurun_out/ncu_expand_sssp_{tag}.ncu-rep")}
    json.dump(res, open(f"profiles/ncu_{tag}.json", "w"), indent=1)
    b = res["bfs_expand_depth3"][0]
    traffic = (b.get("dram__bytes_read.sum") or 0) + (b.get("dram__bytes_write.sum") or 0)
    unit = b.get("dram__bytes_read.sum [unit]", "byte")
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(unit, 1)
    # algorithmic bytes of the captured launch (BFS model: 8 B per edge + 20 B per
    # active vertex), from the per-iteration trace of the same source
    alg_bytes = None
    try:
        tr = json.load(open(f"gpurun_out/trace_{tag}.json"))["bfs"][3]
        alg_bytes = 8 * tr["edges"] + 20 * tr["nF"]
    except (OSError, KeyError, IndexError, ValueError):
        pass
    summ = {"C2": {"dram_bytes_per_launch": traffic * scale,
                   "algorithmic_bytes_of_captured_launch": alg_bytes,
                   "capture": f"profiles/ncu_{tag}.json bfs_expand_depth3 (ncu --set full, BFS depth-3 launch of C2)"}}
    json.dump(summ, open("profiles/expand_ncu_summary.json", "w"), indent=1)
    print(json.dumps(res["launch_list"], indent=1)[:1500])
    print(json.dumps(res["bfs_expand_depth3"], indent=1)[:2500])
