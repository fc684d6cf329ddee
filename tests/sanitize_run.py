"""Small traversal set for compute-sanitizer (memcheck / racecheck / synccheck / initcheck).

Usage: compute-sanitizer --tool <tool> python tests/sanitize_run.py [graph|hostloop]
(lives under tests/ because it checks the results against the oracle)
  hostloop (default): every handle with ETG_HOST_LOOP (kernels launched from the host);
  graph: the shipping CUDA-graph conditional WHILE path (see tools/sanitize_graph_repro.cu
         for the tool's behaviour on conditional nodes without any library code).
Covers BFS/SSSP/CC/SSWP in every mode (UDC off, SMP shared/off, wave Delta, auto
Delta, CC shared shadow labels at K = 4), step A2 (etg_udc_slices) and the
communicator paths (3 ranks as threads: destination partition BFS/SSSP, push
partition SSSP/CC)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import graphgen as gg  # noqa: E402
import oracle  # noqa: E402
import paper_conf_ipps_wangzlg19_b200 as etg  # noqa: E402
from paper_conf_ipps_wangzlg19_b200 import dist as edist  # noqa: E402

mode = sys.argv[1] if len(sys.argv) > 1 else "hostloop"
HL = etg.HOST_LOOP if mode == "hostloop" else 0
U = etg.to_u32_numpy
g = gg.make("T12", device="cuda")
gs = gg.make("T12", device="cuda", symmetric=True, weights=False)
off, col, w = g.to("cpu").numpy()
soff, scol, _ = gs.to("cpu").numpy()
s = gg.first_source(g)
for flags in [HL, HL | etg.SMP_SHARED, HL | etg.NO_UDC, HL | etg.NO_SMP]:
    o, c, ww, fl = etg.csr_to_device(g.off, g.col, g.w)
    G = etg.Graph(o, c, ww, n=g.n, flags=fl | flags, validate=True)
    assert np.array_equal(U(G.bfs(s)[0]), oracle.bfs(off, col, s))
    assert np.array_equal(U(G.sssp(s)[0]), oracle.sssp(off, col, w, s))
    assert np.array_equal(U(G.sswp(s)[0]), oracle.sswp(off, col, w, s))
    G2 = etg.Graph(o, c, ww, n=g.n, flags=fl | flags, sssp_delta=8)
    assert np.array_equal(U(G2.sssp(s)[0]), oracle.sssp(off, col, w, s))
    o2, c2, _, fl2 = etg.csr_to_device(gs.off, gs.col, None)
    Gs = etg.Graph(o2, c2, None, n=gs.n, flags=fl2 | flags, symmetric=True)
    assert np.array_equal(U(Gs.cc()[0]), oracle.cc(soff, scol))
o, c, ww, fl = etg.csr_to_device(g.off, g.col, g.w)
etg.Graph(o, c, ww, n=g.n, flags=fl).udc_slices(torch.arange(0, 100, device="cuda"))
# CC shared shadow label with a small K (many multi-shadow vertices), SSSP wave auto
o2, c2, _, fl2 = etg.csr_to_device(gs.off, gs.col, None)
Gs = etg.Graph(o2, c2, None, n=gs.n, K=4, flags=fl2 | HL, symmetric=True)
assert np.array_equal(U(Gs.cc()[0]), oracle.cc(soff, scol))
Ga = etg.Graph(o, c, ww, n=g.n, flags=fl | HL, sssp_delta="auto")
assert np.array_equal(U(Ga.sssp(s)[0]), oracle.sssp(off, col, w, s))
print(f"sanitize run ({mode}): single handle ok", flush=True)

# communicator paths: 3 ranks as threads of this process
gc = g.to("cpu")
parts = edist.local_partitions(gc.off, gc.col, gc.w, gc.n, 3, sssp_delta="auto")
for alg, exp in ((etg.BFS, oracle.bfs(off, col, s)), (etg.SSSP, oracle.sssp(off, col, w, s))):
    lab, _ = edist.run_local(parts, alg, s)
    assert np.array_equal(U(lab), exp)
parts = edist.local_partitions(gc.off, gc.col, gc.w, gc.n, 3, exchange="push")
lab, _ = edist.run_local(parts, etg.SSSP, s)
assert np.array_equal(U(lab), oracle.sssp(off, col, w, s))
gsc = gs.to("cpu")
parts = edist.local_partitions(gsc.off, gsc.col, None, gsc.n, 3, exchange="push", symmetric=True)
lab, _ = edist.run_local(parts, etg.CC, 0)
assert np.array_equal(U(lab), oracle.cc(soff, scol))
print(f"sanitize run ({mode}): partitions ok", flush=True)
