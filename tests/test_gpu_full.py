"""Parity at BASELINE.json's full sizes, in the launch configuration bench.py
times (CUDA-graph loop, K = 32, default flags, SSSP with sssp_delta="auto" --
bench.py's default schedule): C2 (the bench workload) and C3
(LiveJournal-shaped, UDC on and off).  The paper's own SSSP schedule (Delta =
0) is checked beside it.  The single-threaded oracle finishes these in
seconds, so the comparison is complete (all n labels), not sampled."""
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
    """The bench's handle (bench.py mk(): K = 32, flags 0, sssp_delta "auto")
    and its sources (gg.sample_sources(g, 16, 4242), the first three)."""
    off, col, w = c2.to("cpu").numpy()
    G = to_etg(c2, sssp_delta="auto")
    for s in gg.sample_sources(c2, 16, 4242)[:3]:
        np.testing.assert_array_equal(U32(G.bfs(s)[0]), oracle.bfs(off, col, s))
        np.testing.assert_array_equal(U32(G.sssp(s)[0]), oracle.sssp(off, col, w, s), err_msg=f"auto s={s}")
    s = gg.first_source(c2)
    np.testing.assert_array_equal(U32(G.sswp(s)[0]), oracle.sswp(off, col, w, s))
    # the paper's schedule (Proc. 1: every improved vertex active next iteration)
    Gp = to_etg(c2, sssp_delta=0)
    np.testing.assert_array_equal(U32(Gp.sssp(s)[0]), oracle.sssp(off, col, w, s), err_msg="paper schedule")


def test_c2_cc():
    gs = gg.make("C2", device="cuda", symmetric=True, weights=False)
    soff, scol, _ = gs.to("cpu").numpy()
    G = to_etg(gs, symmetric=True)
    np.testing.assert_array_equal(U32(G.cc()[0]), oracle.cc(soff, scol))


@pytest.mark.parametrize("flags", [0, 2])
def test_c3_lj_shaped(flags):
    g = gg.make("C3", device="cuda")
    off, col, w = g.to("cpu").numpy()
    G = to_etg(g, flags=flags, sssp_delta="auto")
    for s in [gg.first_source(g)] + gg.sample_sources(g, 16, 4242)[:1]:
        np.testing.assert_array_equal(U32(G.bfs(s)[0]), oracle.bfs(off, col, s))
        np.testing.assert_array_equal(U32(G.sssp(s)[0]), oracle.sssp(off, col, w, s), err_msg=f"auto s={s}")


@pytest.mark.parametrize("exchange", ["dest", "push"])
def test_c2_partitioned_4way(c2, exchange):
    """The partitioned path at the bench size: 4 communicator ranks (threads,
    one GPU), SSSP in the bench's schedule (auto Delta, resolved from the
    global sums) and CC; owned slices concatenated = the oracle, all n."""
    from paper_conf_ipps_wangzlg19_b200 import dist as edist
    off, col, w = c2.to("cpu").numpy()
    s = gg.sample_sources(c2, 16, 4242)[0]
    parts = edist.local_partitions(c2.off, c2.col, c2.w, c2.n, 4, exchange=exchange, sssp_delta="auto")
    labels, st = edist.run_local(parts, etg.SSSP, s)
    np.testing.assert_array_equal(U32(labels), oracle.sssp(off, col, w, s))
    if exchange == "dest":
        labels, _ = edist.run_local(parts, etg.BFS, s)
        np.testing.assert_array_equal(U32(labels), oracle.bfs(off, col, s))
    for p in parts:
        p.close()
    del parts
    gs = gg.make("C2", device="cuda", symmetric=True, weights=False)
    soff, scol, _ = gs.to("cpu").numpy()
    parts = edist.local_partitions(gs.off, gs.col, None, gs.n, 4, exchange=exchange, symmetric=True)
    labels, _ = edist.run_local(parts, etg.CC, 0)
    np.testing.assert_array_equal(U32(labels), oracle.cc(soff, scol))
