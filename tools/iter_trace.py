"""Per-iteration trace of one traversal: for every iteration, the active-set
size, shadows, edges expanded and the CUDA-event time of the expand and the
scan launch (step-wise ABI, so each launch is bracketed on the handle's
stream).  Usage: python tools/iter_trace.py --config C2 --algs bfs,sssp,cc"""
import argparse
import ctypes
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import graphgen as gg  # noqa: E402
import paper_conf_ipps_wangzlg19_b200 as etg  # noqa: E402
from paper_conf_ipps_wangzlg19_b200 import lib, _check, _ptr  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="C2")
ap.add_argument("--algs", default="bfs,sssp,cc")
ap.add_argument("--K", type=int, default=32)
ap.add_argument("--flags", type=int, default=0)
ap.add_argument("--delta", type=int, default=0)
ap.add_argument("--json", default="")
a = ap.parse_args()
dev = torch.device("cuda:0")
algs = a.algs.split(",")
ALG = {"bfs": etg.BFS, "sssp": etg.SSSP, "cc": etg.CC, "sswp": etg.SSWP}
out = {}
for alg in algs:
    sym = alg == "cc"
    g = gg.make(a.config, device=dev, symmetric=sym, weights=alg in ("sssp", "sswp"))
    src = 0 if sym else gg.sample_sources(g, 1, 4242)[0]
    o, c, w, fl = etg.csr_to_device(g.off, g.col, g.w, device=dev)
    G = etg.Graph(o, c, w, n=g.n, K=a.K, flags=a.flags | fl, symmetric=sym, sssp_delta=a.delta)
    lab = torch.empty(g.n, dtype=torch.int32, device=dev)
    L = lib()
    cnt = (ctypes.c_uint64 * 6)()
    rows = []
    for rep in range(2):                       # rep 0 warms up (graph/attribute setup)
        rows = []
        na = ctypes.c_uint32()
        _check(L.etg_step_begin(G._h, ALG[alg], src, _ptr(lab), ctypes.byref(na)), "begin")
        L.etg_debug_counters(G._h, cnt)
        prev_edges = cnt[3]
        while na.value:
            nF, nsh = cnt[1], cnt[2]
            e0, e1, e2 = (torch.cuda.Event(enable_timing=True) for _ in range(3))
            e0.record()
            _check(L.etg_step_expand(G._h), "expand")
            e1.record()
            _check(L.etg_step_scan(G._h, ctypes.byref(na)), "scan")
            e2.record()
            torch.cuda.synchronize()
            L.etg_debug_counters(G._h, cnt)
            rows.append({"depth": int(cnt[0]) - 1, "nF": int(nF), "shadows": int(nsh),
                         "edges": int(cnt[3] - prev_edges), "activated": int(na.value),
                         "expand_us": e0.elapsed_time(e1) * 1e3, "scan_us": e1.elapsed_time(e2) * 1e3})
            prev_edges = cnt[3]
        st = etg.Stats()
        _check(L.etg_step_end(G._h, ctypes.byref(st)), "end")
    tot_e = sum(r["expand_us"] for r in rows)
    tot_s = sum(r["scan_us"] for r in rows)
    edges = sum(r["edges"] for r in rows)
    print(f"== {alg} on {a.config}: {len(rows)} iterations, expand {tot_e:.0f} us, scan {tot_s:.0f} us, "
          f"edges {edges/1e6:.1f} M ({edges/max(tot_e,1e-9)/1e3:.1f} G edges/s in expand)")
    for r in rows:
        rate = r["edges"] / max(r["expand_us"], 1e-9) / 1e3
        print(f"  d{r['depth']:3d} nF {r['nF']:9d} sh {r['shadows']:9d} edges {r['edges']:10d} "
              f"act {r['activated']:9d} exp {r['expand_us']:8.1f} us ({rate:6.1f} G/s) scan {r['scan_us']:7.1f} us")
    out[alg] = rows
    del G
    torch.cuda.empty_cache()
if a.json:
    json.dump(out, open(a.json, "w"), indent=1)
