import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch, graphgen as gg, paper_conf_ipps_wangzlg19_b200 as etg
g = gg.make(sys.argv[1] if len(sys.argv) > 1 else "C2", device="cuda")
s = gg.sample_sources(g, 1, 4242)[0]
o, c, w, fl = etg.csr_to_device(g.off, g.col, g.w, device="cuda")
for dl in [0, 8, 16, 32, 64, 256]:
    G = etg.Graph(o, c, w, n=g.n, flags=fl, sssp_delta=dl)
    G.sssp(s)
    _, st = G.sssp(s)
    print(f"delta={dl:4d} iters={st.iterations:4d} edges={st.edges_processed/1e6:8.1f}M acts={st.activations/1e6:6.2f}M ms={st.ms:.3f}")
