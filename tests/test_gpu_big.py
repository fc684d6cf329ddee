"""Parity at the two billion-edge configs, in the bench's launch configuration.

C4 (Twitter-shaped, ~1.5 B edges, SSSP with UDC) in the bench's SSSP
schedule (sssp_delta="auto", Delta = 6 here): the GPU distances must equal
the oracle's Dijkstra distances for all n vertices (and pass the device-side
shortest-path certificate, itself pinned in tests/test_oracle.py), and the GPU
BFS depths must equal the oracle's.
C5 (RMAT scale 28, ~4.3 B edges, BFS): the GPU depths -- single partition and
a 2-way destination partition over the library's communicator -- must equal
the oracle's for all n vertices.  These take minutes (generation + a
single-threaded oracle pass over billions of edges)."""
import numpy as np
import pytest
import torch

import graphgen as gg
import oracle
from etg_testutil import sssp_certificate_gpu, to_etg

pytestmark = [pytest.mark.gpu, pytest.mark.slow]
etg = pytest.importorskip("paper_conf_ipps_wangzlg19_b200")
from paper_conf_ipps_wangzlg19_b200 import dist as edist  # noqa: E402
U32 = etg.to_u32_numpy


def test_c4_sssp_oracle_and_bfs():
    g = gg.make("C4", device="cuda")
    s = gg.first_source(g)
    G = to_etg(g, sssp_delta="auto")
    dist, st = G.sssp(s)
    assert sssp_certificate_gpu(g, s, dist) is None
    depth, _ = G.bfs(s)
    G.close()
    got_d, got_b = U32(dist), U32(depth)
    off = g.off.cpu().numpy().astype(np.uint64)
    col = g.col.to(torch.int32).cpu().numpy().view(np.uint32)
    w = g.w.to(torch.int32).cpu().numpy().view(np.uint32)
    del g, G, dist, depth
    torch.cuda.empty_cache()
    np.testing.assert_array_equal(got_b, oracle.bfs(off, col, s))
    np.testing.assert_array_equal(got_d, oracle.sssp(off, col, w, s))


def test_c5_bfs_single_and_partitioned():
    g = gg.make("C5", device="cuda", weights=False)
    s = gg.sample_sources(g, 1, 28)[0]
    G = to_etg(g)
    depth, st = G.bfs(s)
    got = U32(depth)
    G.close()
    del G, depth
    torch.cuda.empty_cache()
    # 2-way destination partition: two communicator ranks (threads) on this GPU
    parts = edist.local_partitions(g.off, g.col, None, g.n, 2)
    labels, pst = edist.run_local(parts, etg.BFS, s)
    got_p = U32(labels)
    for p in parts:
        p.close()
    del parts, labels
    off = g.off.cpu().numpy().astype(np.uint64)
    col = g.col.to(torch.int32).cpu().numpy().view(np.uint32)
    del g
    torch.cuda.empty_cache()
    exp = oracle.bfs(off, col, s)
    np.testing.assert_array_equal(got, exp)
    np.testing.assert_array_equal(got_p, exp)
