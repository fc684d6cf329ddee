"""Parity at the two billion-edge configs, in the bench's launch configuration.

C4 (Twitter-shaped, ~1.4 B edges, SSSP with UDC): the GPU distances must pass
the shortest-path certificate (checked on the device over every edge), and
the GPU BFS depths must equal the oracle's for all n vertices.
C5 (RMAT scale 28, ~4.3 B edges, BFS): the GPU depths -- single partition and
a 2-way destination partition driven by the multi-GPU driver -- must equal
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


def test_c4_sssp_certificate_and_bfs():
    g = gg.make("C4", device="cuda")
    s = gg.first_source(g)
    G = to_etg(g)
    dist, st = G.sssp(s)
    assert sssp_certificate_gpu(g, s, dist) is None
    depth, _ = G.bfs(s)
    G.close()
    off = g.off.cpu().numpy().astype(np.uint64)
    col = g.col.to(torch.int32).cpu().numpy().view(np.uint32)
    del g
    torch.cuda.empty_cache()
    np.testing.assert_array_equal(U32(depth), oracle.bfs(off, col, s))


def test_c5_bfs_single_and_partitioned():
    g = gg.make("C5", device="cuda", weights=False)
    s = gg.sample_sources(g, 1, 28)[0]
    G = to_etg(g)
    depth, st = G.bfs(s)
    got = U32(depth)
    G.close()
    del G, depth
    torch.cuda.empty_cache()
    # 2-way destination partition through the multi-GPU driver (loopback)
    bounds = edist.partition_ranges(g.off, g.col, g.n, 2)
    engines = []
    for r in range(2):
        loff, lcol, _ = edist.partition_csr(g.off, g.col, None, g.n, bounds[r], bounds[r + 1])
        o, c, _, fl = etg.csr_to_device(loff, lcol, None, device="cuda")
        del loff, lcol
        engines.append(edist.CudaEngine(etg.Graph(o, c, None, n=g.n, flags=fl)))
    labels, pst = edist.run_partitions(engines, edist.LoopbackGroup(), etg.BFS, s)
    got_p = U32(labels)
    del engines, labels
    off = g.off.cpu().numpy().astype(np.uint64)
    col = g.col.to(torch.int32).cpu().numpy().view(np.uint32)
    del g
    torch.cuda.empty_cache()
    exp = oracle.bfs(off, col, s)
    np.testing.assert_array_equal(got, exp)
    np.testing.assert_array_equal(got_p, exp)
