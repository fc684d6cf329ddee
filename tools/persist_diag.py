"""Persistent loop vs CUDA-graph loop on one config: per-call device time and,
for the persistent loop, the %globaltimer split into expand / scan phases.
usage: python tools/persist_diag.py [--config C2] [--tunes 0,1024] [--delta 0]"""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import graphgen as gg  # noqa: E402
import paper_conf_ipps_wangzlg19_b200 as etg  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="C2")
ap.add_argument("--tunes", default="0,1024")
ap.add_argument("--algs", default="bfs,sssp,cc")
ap.add_argument("--delta", type=int, default=0)
ap.add_argument("--reps", type=int, default=5)
a = ap.parse_args()
dev = torch.device("cuda:0")
g = gg.make(a.config, device=dev)
gs = gg.make(a.config, device=dev, symmetric=True, weights=False)
src = gg.sample_sources(g, 1, 4242)[0]
o, c, w, fl = etg.csr_to_device(g.off, g.col, g.w, device=dev)
o2, c2, _, fl2 = etg.csr_to_device(gs.off, gs.col, None, device=dev)
for tune in a.tunes.split(","):
    # "prof": the separate kernels with CUDA events around each launch (ETG_PROFILE)
    pf = etg.PROFILE if tune == "prof" else 0
    os.environ["ETG_TUNE"] = "0" if tune == "prof" else tune
    G = etg.Graph(o, c, w, n=g.n, flags=fl | pf, sssp_delta=a.delta)
    Gs = etg.Graph(o2, c2, None, n=gs.n, flags=fl2 | pf, symmetric=True)
    for alg in a.algs.split(","):
        rows = []
        for r in range(a.reps + 2):
            if alg == "cc":
                _, st = Gs.cc()
            else:
                _, st = G.run({"bfs": etg.BFS, "sssp": etg.SSSP, "sswp": etg.SSWP}[alg], src)
            rows.append(st.asdict())
        rows = rows[2:]
        mean = lambda k: sum(r[k] for r in rows) / len(rows)  # noqa: E731
        print(f"tune={tune:5s} {alg:5s} ms {mean('ms'):.3f} expand {mean('expand_ms'):.3f} scan {mean('scan_ms'):.3f} "
              f"iters {rows[-1]['iterations']} edges {rows[-1]['edges_processed']}")
    G.close()
    Gs.close()
