"""Time one expand iteration of C2 under tune variants (etg_debug_expand_replay)."""
import argparse, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import graphgen as gg
import paper_conf_ipps_wangzlg19_b200 as etg
ap = argparse.ArgumentParser()
ap.add_argument("--config", default="C2")
ap.add_argument("--alg", default="bfs")
ap.add_argument("--depths", default="3,4")
ap.add_argument("--tunes", default="0,16,32")
ap.add_argument("--K", type=int, default=32)
ap.add_argument("--flags", type=int, default=0)
a = ap.parse_args()
dev = torch.device("cuda:0")
alg = {"bfs": etg.BFS, "sssp": etg.SSSP, "cc": etg.CC, "sswp": etg.SSWP}[a.alg]
g = gg.make(a.config, device=dev, weights=a.alg in ("sssp", "sswp"), symmetric=(a.alg == "cc"))
src = gg.sample_sources(g, 1, 4242)[0]
o, c, w, fl = etg.csr_to_device(g.off, g.col, g.w, device=dev)
G = etg.Graph(o, c, w, n=g.n, K=a.K, flags=a.flags | fl, symmetric=(a.alg == "cc"))
for dpt in [int(x) for x in a.depths.split(",")]:
    for t in [int(x) for x in a.tunes.split(",")]:
        ms, edges, nact = G.debug_expand_replay(alg, src, dpt, t, reps=5)
        print(f"{a.alg} depth={dpt} tune={t:3d} nF={nact:8d} edges={edges:9d} ms={ms:8.3f}  G edges/s={edges/ms/1e6:7.1f}")
