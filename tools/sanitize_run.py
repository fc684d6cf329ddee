"""Small traversal set for compute-sanitizer (memcheck / racecheck / synccheck / initcheck)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import graphgen as gg, oracle, paper_conf_ipps_wangzlg19_b200 as etg
g = gg.make("T12", device="cuda")
gs = gg.make("T12", device="cuda", symmetric=True, weights=False)
off, col, w = g.to("cpu").numpy()
s = gg.first_source(g)
for flags in [0, etg.HOST_LOOP, etg.SMP_SHARED, etg.NO_UDC]:
    o, c, ww, fl = etg.csr_to_device(g.off, g.col, g.w)
    G = etg.Graph(o, c, ww, n=g.n, flags=fl | flags, validate=True)
    assert np.array_equal(etg.to_u32_numpy(G.bfs(s)[0]), oracle.bfs(off, col, s))
    assert np.array_equal(etg.to_u32_numpy(G.sssp(s)[0]), oracle.sssp(off, col, w, s))
    G2 = etg.Graph(o, c, ww, n=g.n, flags=fl | flags, sssp_delta=8)
    assert np.array_equal(etg.to_u32_numpy(G2.sssp(s)[0]), oracle.sssp(off, col, w, s))
    o2, c2, _, fl2 = etg.csr_to_device(gs.off, gs.col, None)
    Gs = etg.Graph(o2, c2, None, n=gs.n, flags=fl2 | flags, symmetric=True)
    Gs.cc()
o, c, ww, fl = etg.csr_to_device(g.off, g.col, g.w)
ids = etg.Graph(o, c, ww, n=g.n, flags=fl).udc_slices(torch.arange(0, 100, device="cuda"))
print("sanitize run ok")
