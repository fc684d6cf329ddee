import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch, graphgen as gg, paper_conf_ipps_wangzlg19_b200 as etg
g = gg.make("C2", device="cuda")
gs = gg.make("C2", device="cuda", symmetric=True, weights=False)
s = gg.sample_sources(g, 1, 4242)[0]
o, c, w, fl = etg.csr_to_device(g.off, g.col, g.w, device="cuda")
o2, c2, _, fl2 = etg.csr_to_device(gs.off, gs.col, None, device="cuda")
for name, mk, run in [
        ("bfs", lambda f, d: etg.Graph(o, c, w, n=g.n, flags=fl | f, sssp_delta=d), lambda G: G.bfs(s)),
        ("sssp d0", lambda f, d: etg.Graph(o, c, w, n=g.n, flags=fl | f), lambda G: G.sssp(s)),
        ("sssp d16", lambda f, d: etg.Graph(o, c, w, n=g.n, flags=fl | f, sssp_delta=16), lambda G: G.sssp(s)),
        ("cc", lambda f, d: etg.Graph(o2, c2, None, n=g.n, flags=fl2 | f, symmetric=True), lambda G: G.cc())]:
    Gp = mk(etg.PROFILE, 0); run(Gp); _, st = run(Gp)
    Gg = mk(0, 0); run(Gg); _, sg = run(Gg)
    print(f"{name:9s} graph-mode call {sg.ms:.3f} ms | host-loop call {st.ms:.3f}: expand {st.expand_ms:.3f} "
          f"({st.expand_launches} launches) scan {st.scan_ms:.3f} | iters {st.iterations} edges {st.edges_processed/1e6:.1f}M")
