"""Parity at BASELINE.json's full sizes, in the launch configuration bench.py
times (CUDA-graph loop, K = 32, default flags): C2 (the bench workload) and
C3 (LiveJournal-shaped, UDC on and off).  The single-threaded oracle finishes
these in seconds, so the comparison is complete (all n labels), not sampled."""
import numpy as np
import pytest
import torch

import graphgen as gg
import oracle
from etg_testutil import to_etg

pytestmark = pytest.mark.gpu
etg = pytest.importorskip("paper_conf_ipps_wangzlg19_b200")
U32 = etg.to_u32_numpy


@pytest.fixture(scope="module")
def c2():
    return gg.make("C2", device="cuda")


def test_c2_bfs_sssp_sswp(c2):
    off, col, w = c2.to("cpu").numpy()
    G = to_etg(c2)
    for s in gg.sample_sources(c2, 2, 4242):
        np.testing.assert_array_equal(U32(G.bfs(s)[0]), oracle.bfs(off, col, s))
        np.testing.assert_array_equal(U32(G.sssp(s)[0]), oracle.sssp(off, col, w, s))
    s = gg.first_source(c2)
    np.testing.assert_array_equal(U32(G.sswp(s)[0]), oracle.sswp(off, col, w, s))


def test_c2_cc():
    gs = gg.make("C2", device="cuda", symmetric=True, weights=False)
    soff, scol, _ = gs.to("cpu").numpy()
    G = to_etg(gs, symmetric=True)
    np.testing.assert_array_equal(U32(G.cc()[0]), oracle.cc(soff, scol))


@pytest.mark.parametrize("flags", [0, 2])
def test_c3_lj_shaped(flags):
    g = gg.make("C3", device="cuda")
    off, col, w = g.to("cpu").numpy()
    G = to_etg(g, flags=flags)
    s = gg.first_source(g)
    np.testing.assert_array_equal(U32(G.bfs(s)[0]), oracle.bfs(off, col, s))
    np.testing.assert_array_equal(U32(G.sssp(s)[0]), oracle.sssp(off, col, w, s))


def test_c2_push_exchange_4way(c2):
    """NEXT-3 at the bench size: SSSP and CC on a 4-way SOURCE partition with the
    push exchange (auto: sparse all-to-all or dense reduce per iteration), P
    engines on one GPU (LoopbackGroup); owned slices assembled = the oracle."""
    from paper_conf_ipps_wangzlg19_b200 import dist as edist
    P = 4

    def run(g, alg, s):
        bounds = edist.partition_ranges(g.off, g.col, g.n, P, by="out")
        engs = []
        for r in range(P):
            loff, lcol, lw = edist.partition_csr_src(g.off, g.col, g.w, g.n, bounds[r], bounds[r + 1])
            o, c, w, fl = etg.csr_to_device(loff, lcol, lw, device="cuda")
            engs.append(edist.CudaEngine(etg.Graph(o, c, w, n=g.n, flags=fl, symmetric=g.symmetric)))
        _, _, used = edist.run_push(engs, edist.LoopbackGroup(), alg, s, bounds, list(range(P)))
        return np.concatenate([U32(e.labels)[bounds[r]:bounds[r + 1]] for r, e in enumerate(engs)]), used

    off, col, w = c2.to("cpu").numpy()
    s = gg.sample_sources(c2, 1, 4242)[0]
    got, used = run(c2, etg.SSSP, s)
    np.testing.assert_array_equal(got, oracle.sssp(off, col, w, s))
    assert used["sparse"] > 0 and used["dense"] > 0          # both exchanges exercised at this size
    gs = gg.make("C2", device="cuda", symmetric=True, weights=False)
    soff, scol, _ = gs.to("cpu").numpy()
    got, _ = run(gs, etg.CC, 0)
    np.testing.assert_array_equal(got, oracle.cc(soff, scol))


def test_c2_push_p2p_4way(c2):
    """The fused push exchange at the bench size: 4 source partitions on one GPU,
    each expand reducing straight into the owners' label arrays."""
    from paper_conf_ipps_wangzlg19_b200 import dist as edist
    P = 4
    bounds = edist.partition_ranges(c2.off, c2.col, c2.n, P, by="out")
    engs = []
    for r in range(P):
        loff, lcol, lw = edist.partition_csr_src(c2.off, c2.col, c2.w, c2.n, bounds[r], bounds[r + 1])
        o, c, w, fl = etg.csr_to_device(loff, lcol, lw, device="cuda")
        engs.append(edist.CudaEngine(etg.Graph(o, c, w, n=c2.n, flags=fl)))
    for r, e in enumerate(engs):
        e.set_peers(bounds, r, [x.labels.data_ptr() for x in engs])
    s = gg.sample_sources(c2, 1, 4242)[0]
    edist.run_push(engs, edist.LoopbackGroup(), etg.SSSP, s, bounds, list(range(P)), "p2p")
    off, col, w = c2.to("cpu").numpy()
    got = np.concatenate([U32(e.labels)[bounds[r]:bounds[r + 1]] for r, e in enumerate(engs)])
    np.testing.assert_array_equal(got, oracle.sssp(off, col, w, s))
