"""Multi-rank path: partitioning and the exchange driver, on the CPU.

* partition properties (every edge in exactly one part, word-aligned ranges,
  in-edge balance);
* the driver with P in-process ranks (LoopbackGroup) and with world_size 2
  over gloo (torch.distributed, 127.0.0.1), each rank a test-only numpy step
  engine (tests/etg_mock_engine.py) -- labels must equal the oracle's.
The CUDA engine through the same driver is covered by tests/test_gpu_dist.py.
"""
import os

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import graphgen as gg
import oracle
from etg_mock_engine import MockEngine
from paper_conf_ipps_wangzlg19_b200 import dist as edist

ALGS = {"bfs": 0, "sssp": 1, "cc": 2, "sswp": 3}


def expected(alg, g, s):
    off, col, w = g.numpy()
    if alg == "bfs":
        return oracle.bfs(off, col, s)
    if alg == "sssp":
        return oracle.sssp(off, col, w, s)
    if alg == "sswp":
        return oracle.sswp(off, col, w, s)
    return oracle.cc(off, col)


def make_parts(g, P):
    bounds = edist.partition_ranges(g.off, g.col, g.n, P)
    parts = []
    for r in range(P):
        loff, lcol, lw = edist.partition_csr(g.off, g.col, g.w, g.n, bounds[r], bounds[r + 1])
        parts.append(MockEngine(loff.numpy(), lcol.numpy(), None if lw is None else lw.numpy(), g.n))
    return bounds, parts


@pytest.mark.parametrize("P", [1, 2, 3, 5])
def test_partition_properties(P):
    g = gg.make("T12")
    bounds = edist.partition_ranges(g.off, g.col, g.n, P)
    assert bounds[0] == 0 and bounds[-1] == g.n and len(bounds) == P + 1
    assert all(b % 32 == 0 for b in bounds[:-1]) and all(a <= b for a, b in zip(bounds, bounds[1:]))
    seen = 0
    indeg = np.bincount(g.col.numpy(), minlength=g.n)
    for r in range(P):
        loff, lcol, lw = edist.partition_csr(g.off, g.col, g.w, g.n, bounds[r], bounds[r + 1])
        assert loff.shape[0] == g.n + 1 and int(loff[-1]) == lcol.shape[0]
        assert torch.all((lcol >= bounds[r]) & (lcol < bounds[r + 1]))
        seen += lcol.shape[0]
        share = indeg[bounds[r]:bounds[r + 1]].sum() / g.m
        assert abs(share - 1 / P) < 0.05
    assert seen == g.m


@pytest.mark.parametrize("gather", [False, True])
@pytest.mark.parametrize("alg", ["bfs", "sssp", "cc", "sswp"])
@pytest.mark.parametrize("P", [2, 3])
def test_loopback_driver_matches_oracle(alg, P, gather):
    """Both exchanges: full-array all-reduce, and the all-gather of owned slices."""
    g = gg.make("T12") if alg != "cc" else gg.make("T12", symmetric=True, weights=False)
    s = gg.first_source(g)
    bounds, parts = make_parts(g, P)
    labels, st = edist.run_partitions(parts, edist.LoopbackGroup(), ALGS[alg], s,
                                      bounds if gather else None)
    np.testing.assert_array_equal(labels.numpy().view(np.uint32), expected(alg, g, s))
    if alg == "bfs":
        assert st.edges_processed == int(np.diff(g.off.numpy())[expected(alg, g, s) != oracle.INF].sum())


@pytest.mark.parametrize("alg", ["bfs", "sssp", "cc", "sswp"])
@pytest.mark.parametrize("P", [2, 3])
def test_dest_p2p_loopback_matches_oracle(alg, P):
    """The fused destination-partition exchange's protocol: each engine
    publishes its owned changes into the peers' copies, no collective."""
    g = gg.make("T12") if alg != "cc" else gg.make("T12", symmetric=True, weights=False)
    s = gg.first_source(g)
    bounds, parts = make_parts(g, P)
    for r, p in enumerate(parts):
        p.set_dest_peers(bounds, r, [q.q for q in parts], [q.labels for q in parts])
    labels, st = edist.run_partitions(parts, edist.LoopbackGroup(), ALGS[alg], s, bounds, "p2p")
    for p in parts:       # every rank holds the full result, as with the all-gather
        np.testing.assert_array_equal(p.labels.numpy().view(np.uint32), expected(alg, g, s))


def _gloo_worker(rank, world, port, alg, out, gather=False):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    g = gg.make("T12") if alg != "cc" else gg.make("T12", symmetric=True, weights=False)
    s = gg.first_source(g)
    bounds = edist.partition_ranges(g.off, g.col, g.n, world)
    loff, lcol, lw = edist.partition_csr(g.off, g.col, g.w, g.n, bounds[rank], bounds[rank + 1])
    eng = MockEngine(loff.numpy(), lcol.numpy(), None if lw is None else lw.numpy(), g.n)
    labels, st = edist.run_partitions([eng], edist.TorchDistGroup(), ALGS[alg], s, bounds if gather else None)
    torch.save(labels, out + f".{rank}")
    dist.destroy_process_group()


@pytest.mark.parametrize("gather", [False, True])
@pytest.mark.parametrize("alg", ["bfs", "sssp", "cc"])
def test_gloo_world2_matches_oracle(alg, gather, tmp_path):
    port = 29500 + (os.getpid() % 1000) + ALGS[alg] + (8 if gather else 0)
    out = str(tmp_path / "labels")
    mp.spawn(_gloo_worker, args=(2, port, alg, out, gather), nprocs=2, join=True)
    g = gg.make("T12") if alg != "cc" else gg.make("T12", symmetric=True, weights=False)
    exp = expected(alg, g, gg.first_source(g))
    for r in range(2):
        got = torch.load(out + f".{r}").numpy().view(np.uint32)
        np.testing.assert_array_equal(got, exp)


# --------------------------------------------------------------------------- #
# NEXT-3: source partition + push exchange (all-to-all of proposals / dense
# reduce onto the owners)
# --------------------------------------------------------------------------- #
def make_src_parts(g, P):
    bounds = edist.partition_ranges(g.off, g.col, g.n, P, by="out")
    parts = []
    for r in range(P):
        loff, lcol, lw = edist.partition_csr_src(g.off, g.col, g.w, g.n, bounds[r], bounds[r + 1])
        parts.append(MockEngine(loff.numpy(), lcol.numpy(), None if lw is None else lw.numpy(), g.n))
    return bounds, parts


def owned(labels_per_rank, bounds):
    return np.concatenate([labels_per_rank[r][bounds[r]:bounds[r + 1]] for r in range(len(bounds) - 1)])


@pytest.mark.parametrize("P", [1, 2, 3, 5])
def test_source_partition_properties(P):
    g = gg.make("T12")
    bounds = edist.partition_ranges(g.off, g.col, g.n, P, by="out")
    assert bounds[0] == 0 and bounds[-1] == g.n and all(b % 32 == 0 for b in bounds[:-1])
    off = g.off.numpy().astype(np.int64)
    seen = 0
    for r in range(P):
        lo, hi = bounds[r], bounds[r + 1]
        loff, lcol, lw = edist.partition_csr_src(g.off, g.col, g.w, g.n, lo, hi)
        loff = loff.numpy()
        assert loff.shape[0] == g.n + 1 and loff[-1] == lcol.shape[0]
        deg = np.diff(loff)
        assert np.all(deg[:lo] == 0) and np.all(deg[hi:] == 0)
        np.testing.assert_array_equal(deg[lo:hi], np.diff(off)[lo:hi])
        np.testing.assert_array_equal(lcol.numpy(), g.col.numpy()[off[lo]:off[hi]])
        np.testing.assert_array_equal(lw.numpy(), g.w.numpy()[off[lo]:off[hi]])
        seen += lcol.shape[0]
        if P > 1:
            assert abs((off[hi] - off[lo]) / g.m - 1 / P) < 0.05
    assert seen == g.m


@pytest.mark.parametrize("mode", ["sparse", "dense", "auto"])
@pytest.mark.parametrize("alg", ["sssp", "cc", "sswp"])
@pytest.mark.parametrize("P", [2, 3])
def test_push_loopback_matches_oracle(alg, P, mode):
    g = gg.make("T12") if alg != "cc" else gg.make("T12", symmetric=True, weights=False)
    s = gg.first_source(g)
    bounds, parts = make_src_parts(g, P)
    _, st, used = edist.run_push(parts, edist.LoopbackGroup(), ALGS[alg], s, bounds, list(range(P)), mode)
    got = owned([p.labels.numpy().view(np.uint32) for p in parts], bounds)
    np.testing.assert_array_equal(got, expected(alg, g, s))
    if mode != "auto":
        assert used[mode] > 0 and sum(used.values()) == used[mode]


@pytest.mark.parametrize("alg", ["sssp", "cc", "sswp"])
@pytest.mark.parametrize("P", [2, 3])
def test_push_p2p_loopback_matches_oracle(alg, P):
    """The fused exchange's driver protocol (expand writes the owners' labels,
    sync + barrier, scan) with the numpy engine writing peers' arrays."""
    g = gg.make("T12") if alg != "cc" else gg.make("T12", symmetric=True, weights=False)
    s = gg.first_source(g)
    bounds, parts = make_src_parts(g, P)
    for r, p in enumerate(parts):
        p.set_peers(bounds, r, [q.labels for q in parts])
    _, st, used = edist.run_push(parts, edist.LoopbackGroup(), ALGS[alg], s, bounds, list(range(P)), "p2p")
    got = owned([p.labels.numpy().view(np.uint32) for p in parts], bounds)
    np.testing.assert_array_equal(got, expected(alg, g, s))
    assert used.get("p2p", 0) > 0 and used["sparse"] == used["dense"] == 0


def test_push_p2p_needs_peers():
    g = gg.make("T12")
    bounds, parts = make_src_parts(g, 2)
    with pytest.raises(edist.EtgError):
        edist.run_push(parts, edist.LoopbackGroup(), ALGS["sssp"], gg.first_source(g), bounds, [0, 1], "p2p")


def test_push_rejects_bfs():
    g = gg.make("T12")
    bounds, parts = make_src_parts(g, 2)
    with pytest.raises(edist.EtgError):
        edist.run_push(parts, edist.LoopbackGroup(), ALGS["bfs"], 0, bounds, [0, 1])


def _gloo_push_worker(rank, world, port, alg, out, mode):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    g = gg.make("T12") if alg != "cc" else gg.make("T12", symmetric=True, weights=False)
    s = gg.first_source(g)
    bounds = edist.partition_ranges(g.off, g.col, g.n, world, by="out")
    loff, lcol, lw = edist.partition_csr_src(g.off, g.col, g.w, g.n, bounds[rank], bounds[rank + 1])
    eng = MockEngine(loff.numpy(), lcol.numpy(), None if lw is None else lw.numpy(), g.n)
    labels, st, used = edist.run_push([eng], edist.TorchDistGroup(), ALGS[alg], s, bounds, [rank], mode)
    torch.save((labels, bounds, used), out + f".{rank}")
    dist.destroy_process_group()


@pytest.mark.parametrize("mode", ["sparse", "dense", "auto"])
@pytest.mark.parametrize("alg", ["sssp", "cc"])
def test_push_gloo_world2_matches_oracle(alg, mode, tmp_path):
    port = 31500 + (os.getpid() % 1000) + 4 * ALGS[alg] + {"sparse": 0, "dense": 1, "auto": 2}[mode]
    out = str(tmp_path / "labels")
    mp.spawn(_gloo_push_worker, args=(2, port, alg, out, mode), nprocs=2, join=True)
    g = gg.make("T12") if alg != "cc" else gg.make("T12", symmetric=True, weights=False)
    exp = expected(alg, g, gg.first_source(g))
    res = [torch.load(out + f".{r}") for r in range(2)]
    bounds = res[0][1]
    got = owned([res[r][0].numpy().view(np.uint32) for r in range(2)], bounds)
    np.testing.assert_array_equal(got, exp)
    assert res[0][2] == res[1][2]                     # both ranks took the same exchange each iteration
