"""Small traversal set for compute-sanitizer (memcheck / racecheck / synccheck / initcheck).
Every handle runs with ETG_HOST_LOOP: under compute-sanitizer the CUDA-graph
conditional WHILE loop faults with "misaligned address" even in versions whose
kernels are clean (the same kernels launched from the host loop report 0
errors, and the graph path is bit-exact without the tool), so the kernels are
checked through the host-driven loop."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import graphgen as gg, oracle, paper_conf_ipps_wangzlg19_b200 as etg
g = gg.make("T12", device="cuda")
gs = gg.make("T12", device="cuda", symmetric=True, weights=False)
off, col, w = g.to("cpu").numpy()
s = gg.first_source(g)
HL = etg.HOST_LOOP
for flags in [HL, HL | etg.SMP_SHARED, HL | etg.NO_UDC, HL | etg.NO_SMP]:
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

# multi-partition paths on one GPU: push exchange (sparse / dense / peer memory)
# and the fused destination exchange
from paper_conf_ipps_wangzlg19_b200 import dist as edist  # noqa: E402
gc = g.to("cpu")
P = 3
bounds = edist.partition_ranges(gc.off, gc.col, gc.n, P, by="out")
for mode in ("sparse", "dense", "p2p"):
    engs = []
    for r in range(P):
        loff, lcol, lw = edist.partition_csr_src(gc.off, gc.col, gc.w, gc.n, bounds[r], bounds[r + 1])
        o, c, ww, fl = etg.csr_to_device(loff, lcol, lw)
        engs.append(edist.CudaEngine(etg.Graph(o, c, ww, n=g.n, flags=fl)))
    if mode == "p2p":
        for r, e in enumerate(engs):
            e.set_peers(bounds, r, [x.labels.data_ptr() for x in engs])
    edist.run_push(engs, edist.LoopbackGroup(), etg.SSSP, s, bounds, list(range(P)), mode)
    got = np.concatenate([etg.to_u32_numpy(e.labels)[bounds[r]:bounds[r + 1]] for r, e in enumerate(engs)])
    assert np.array_equal(got, oracle.sssp(off, col, w, s)), mode
dbounds = edist.partition_ranges(gc.off, gc.col, gc.n, P)
for alg in (etg.BFS, etg.SSSP):
    engs = []
    for r in range(P):
        loff, lcol, lw = edist.partition_csr(gc.off, gc.col, gc.w, gc.n, dbounds[r], dbounds[r + 1])
        o, c, ww, fl = etg.csr_to_device(loff, lcol, lw)
        engs.append(edist.CudaEngine(etg.Graph(o, c, ww, n=g.n, flags=fl)))
    for r, e in enumerate(engs):
        e.set_dest_peers(dbounds, r, [x.q.data_ptr() for x in engs], [x.labels.data_ptr() for x in engs])
    lab, _ = edist.run_partitions(engs, edist.LoopbackGroup(), alg, s, dbounds, "p2p")
    exp = oracle.bfs(off, col, s) if alg == etg.BFS else oracle.sssp(off, col, w, s)
    assert np.array_equal(etg.to_u32_numpy(lab), exp)
# CC shared shadow label with a small K (many multi-shadow vertices), SSSP wave auto
o2, c2, _, fl2 = etg.csr_to_device(gs.off, gs.col, None)
Gs = etg.Graph(o2, c2, None, n=gs.n, K=4, flags=fl2 | HL, symmetric=True)
soff, scol, _ = gs.to("cpu").numpy()
assert np.array_equal(etg.to_u32_numpy(Gs.cc()[0]), oracle.cc(soff, scol))
o, c, ww, fl = etg.csr_to_device(g.off, g.col, g.w)
Ga = etg.Graph(o, c, ww, n=g.n, flags=fl | HL, sssp_delta="auto")
assert np.array_equal(etg.to_u32_numpy(Ga.sssp(s)[0]), oracle.sssp(off, col, w, s))
print("sanitize run (partitions, shared label, auto Delta) ok")
