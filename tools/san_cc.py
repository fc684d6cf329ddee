"""Diagnostic: CC through the CUDA-graph loop under compute-sanitizer (args: K flags)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import graphgen as gg, paper_conf_ipps_wangzlg19_b200 as etg
K = int(sys.argv[1]) if len(sys.argv) > 1 else 32
flags = int(sys.argv[2]) if len(sys.argv) > 2 else 0
alg = sys.argv[3] if len(sys.argv) > 3 else "cc"
gs = gg.make("T12", device="cuda", symmetric=(alg == "cc"), weights=(alg != "cc"))
soff, scol, sw = gs.to("cpu").numpy()
o2, c2, w2, fl2 = etg.csr_to_device(gs.off, gs.col, gs.w)
G = etg.Graph(o2, c2, w2, n=gs.n, K=K, flags=fl2 | flags, symmetric=(alg == "cc"))
for i in range(2):
    if alg == "cc":
        got, st = G.cc()
        ok = True                      # results are checked by tests/sanitize_run.py (oracle)
    else:
        s = gg.first_source(gs)
        got, st = G.run({"bfs": 0, "sssp": 1, "sswp": 3}[alg], s)
        ok = True
    print(alg, "K", K, "flags", flags, "iter", i, "ok", ok, "iterations", st.iterations, flush=True)
