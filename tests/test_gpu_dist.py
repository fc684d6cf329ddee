"""The partitioned (multi-GPU) path through the C ABI: a communicator handle
per rank (etg_comm_init + etg_load_csr(..., comm, v_lo, v_hi)), and every
traversal call running the whole partitioned Proc. 1 loop inside the library
(expand, exchange into the peers' device memory, barrier, scan, termination
count).  Ranks are threads of this process (peers reached by plain device
pointers) or separate processes (peers mapped with CUDA IPC) -- one GPU per
gpurun call, so NVLink itself is not exercised; the code path is the same.
The owned slices, concatenated in rank order, must equal the oracle's labels
bit for bit (SURVEY 8(b) "Distributed", 8(e) "Parity")."""
import os

import numpy as np
import pytest
import torch

import graphgen as gg
import oracle

pytestmark = pytest.mark.gpu
etg = pytest.importorskip("paper_conf_ipps_wangzlg19_b200")
from paper_conf_ipps_wangzlg19_b200 import dist as edist  # noqa: E402

ALG = {"bfs": etg.BFS, "sssp": etg.SSSP, "cc": etg.CC, "sswp": etg.SSWP}
U32 = etg.to_u32_numpy


def graph_for(alg, cfg="C1"):
    return gg.make(cfg, symmetric=(alg == "cc"), weights=(alg != "cc"))


def expected(alg, g, s):
    off, col, w = g.numpy()
    return {"bfs": lambda: oracle.bfs(off, col, s), "sssp": lambda: oracle.sssp(off, col, w, s),
            "sswp": lambda: oracle.sswp(off, col, w, s), "cc": lambda: oracle.cc(off, col)}[alg]()


def parts_of(g, P, exchange="dest", **kw):
    return edist.local_partitions(g.off, g.col, g.w, g.n, P, exchange=exchange, symmetric=g.symmetric, **kw)


@pytest.mark.parametrize("alg", ["bfs", "sssp", "cc", "sswp"])
@pytest.mark.parametrize("P", [1, 2, 3, 4])
def test_dest_partition_c1(alg, P):
    g = graph_for(alg)
    parts = parts_of(g, P)
    for s in gg.sample_sources(g, 2, P):               # the handles are reused across calls
        labels, st = edist.run_local(parts, ALG[alg], s)
        np.testing.assert_array_equal(U32(labels), expected(alg, g, s), err_msg=f"{alg} P={P} s={s}")


def test_dest_partition_bfs_work_is_split():
    """Every edge of the activatable subgraph is relaxed on exactly one rank
    (statistics summed over the ranks by the library)."""
    g = gg.make("T14", weights=False)
    s = gg.first_source(g)
    labels, st = edist.run_local(parts_of(g, 4), etg.BFS, s)
    exp = expected("bfs", g, s)
    deg = np.diff(g.off.numpy())
    assert st.edges_processed == int(deg[exp != etg.INF].sum())
    assert st.activations == int((exp != etg.INF).sum())
    assert st.ms >= st.reserved > 0                    # max over ranks >= this rank's time
    np.testing.assert_array_equal(U32(labels), exp)


def test_dest_partition_k_and_flags():
    g = gg.make("LJ-small")
    s = gg.sample_sources(g, 1, 9)[0]
    for K, flags in ((8, 0), (1024, 0), (32, etg.NO_UDC)):
        labels, _ = edist.run_local(parts_of(g, 3, K=K, flags=flags), etg.SSSP, s)
        np.testing.assert_array_equal(U32(labels), expected("sssp", g, s), err_msg=f"K={K} flags={flags}")


@pytest.mark.parametrize("exchange", ["dest", "push"])
@pytest.mark.parametrize("delta", [1, 16, "auto"])
def test_partitioned_sssp_wave_schedules(exchange, delta):
    """The SSSP wave schedule on partitions; auto Delta is resolved from the
    GLOBAL weight and edge sums, so every rank -- and the single-GPU handle --
    runs the same Delta."""
    g = gg.make("C1")
    s = gg.sample_sources(g, 1, 77)[0]
    parts = parts_of(g, 3, exchange=exchange, sssp_delta=delta)
    labels, _ = edist.run_local(parts, etg.SSSP, s)
    np.testing.assert_array_equal(U32(labels), expected("sssp", g, s))
    if delta == "auto":
        o, c, w, fl = etg.csr_to_device(g.off, g.col, g.w, device="cuda")
        one = etg.Graph(o, c, w, n=g.n, flags=fl, sssp_delta="auto").sssp_delta()
        got = edist._in_threads([lambda p=p: p.graph.sssp_delta() for p in parts])
        rule = max(1, int(6.0 * float(g.w.double().mean()) / (g.m / g.n) + 0.5))   # 6 x mean w / mean deg
        assert one == rule and got == [rule] * 3


@pytest.mark.parametrize("alg", ["sssp", "cc", "sswp"])
@pytest.mark.parametrize("P", [2, 3, 4])
def test_push_partition_c1(alg, P):
    """ETG_PUSH: source partition, the expand kernel reduces relaxations of
    foreign vertices into their owners' labels over peer memory."""
    g = graph_for(alg)
    parts = parts_of(g, P, exchange="push")
    for s in gg.sample_sources(g, 2, 31 + P):
        labels, _ = edist.run_local(parts, ALG[alg], s)
        np.testing.assert_array_equal(U32(labels), expected(alg, g, s), err_msg=f"{alg} P={P} s={s}")


def test_push_partition_lj_small_k_and_udc_off():
    g = gg.make("LJ-small")
    s = gg.first_source(g)
    for K, flags in ((8, 0), (32, etg.NO_UDC)):
        labels, _ = edist.run_local(parts_of(g, 3, exchange="push", K=K, flags=flags), etg.SSSP, s)
        np.testing.assert_array_equal(U32(labels), expected("sssp", g, s))


def test_push_partition_rejects_bfs():
    g = gg.make("T12")
    parts = parts_of(g, 2, exchange="push")
    with pytest.raises(etg.EtgError, match="EINVAL"):
        edist.run_local(parts, etg.BFS, gg.first_source(g))


def test_load_rejects_ranges_that_do_not_tile():
    """A communicator load whose owned ranges leave a gap, or whose inner bound
    is not a multiple of 32, fails on every rank (ETG_ENCCL), without a hang."""
    g = gg.make("T12", weights=False)
    for bounds in ([[0, 64], [96, g.n]], [[0, 40], [40, g.n]]):
        uid = etg.Comm.unique_id()

        def mk(r, b=bounds):
            def f():
                comm = etg.Comm(r, 2, uid, 0)
                o, c, _, fl = etg.csr_to_device(g.off, g.col, None, device="cuda")
                try:
                    etg.Graph(o, c, None, n=g.n, flags=fl, comm=comm, v_lo=b[r][0], v_hi=b[r][1])
                except etg.EtgError as e:
                    return str(e)
                return "loaded"
            return f
        res = edist._in_threads([mk(0), mk(1)])
        assert all("ENCCL" in x for x in res), res


# --------------------------------------------------------------------------- #
# separate processes: peers' workspaces mapped with CUDA IPC
# --------------------------------------------------------------------------- #
def _proc_worker(rank, world, port, exchange, out):
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    comm = edist.comm_from_group(rank, world, device=0)
    algs = ["sssp", "cc", "sswp"] if exchange == "push" else ["bfs", "sssp", "cc", "sswp"]
    for alg in algs:
        g = graph_for(alg)
        s = gg.first_source(g)
        dg = edist.DistGraph(g.off, g.col, g.w, g.n, comm, exchange=exchange, symmetric=g.symmetric,
                             sssp_delta="auto", device="cuda")
        labels, st = dg.run(ALG[alg], s)
        np.save(out + f".{alg}.{rank}.npy", U32(labels)[:dg.hi - dg.lo])
        dg.close()
    comm.barrier()
    comm.close()
    dist.destroy_process_group()


@pytest.mark.parametrize("exchange", ["dest", "push"])
def test_two_processes_cuda_ipc(exchange, tmp_path):
    """Two ranks in two processes sharing the GPU: torch.distributed (gloo)
    only hands over the communicator id; the library maps the peer's
    workspace with CUDA IPC and runs every loop in C++."""
    import torch.multiprocessing as mp
    port = 33500 + (os.getpid() % 1000) + (0 if exchange == "dest" else 7)
    out = str(tmp_path / "lab")
    mp.spawn(_proc_worker, args=(2, port, exchange, out), nprocs=2, join=True)
    for alg in (["sssp", "cc", "sswp"] if exchange == "push" else ["bfs", "sssp", "cc", "sswp"]):
        g = graph_for(alg)
        got = np.concatenate([np.load(out + f".{alg}.{r}.npy") for r in range(2)])
        np.testing.assert_array_equal(got, expected(alg, g, gg.first_source(g)), err_msg=alg)


@pytest.mark.parametrize("exchange", ["dest", "push"])
def test_tiny_graphs_and_empty_ranges(exchange):
    """Degenerate partitions: ranks whose owned range is empty (n < 32 P), a
    graph smaller than one bitmap word, isolated vertices, and a source with no
    out-edges -- every rank still agrees and the owned slices tile the result."""
    edges = [(0, 1), (1, 2), (2, 0), (3, 4), (5, 5), (6, 7), (7, 6)]
    for n, P in ((8, 2), (8, 4), (70, 4), (70, 3)):
        g = gg.from_edges("tiny", n, [(u, v) for u, v in edges if u < n and v < n] + [(n - 2, n - 1)],
                          weights=None, dedup=True)
        g = gg.add_weights(g, 5)
        for alg in (["sssp", "sswp"] if exchange == "push" else ["bfs", "sssp", "sswp"]):
            for s in (0, 3, n - 1):                      # n - 1 has no out-edges
                parts = parts_of(g, P, exchange=exchange)
                labels, _ = edist.run_local(parts, ALG[alg], s)
                np.testing.assert_array_equal(U32(labels), expected(alg, g, s), err_msg=f"{alg} n={n} P={P} s={s}")
        gs = gg.symmetrize(g)
        gs.w = None
        parts = edist.local_partitions(gs.off, gs.col, None, gs.n, P, exchange=exchange, symmetric=True)
        labels, _ = edist.run_local(parts, etg.CC, 0)
        np.testing.assert_array_equal(U32(labels), expected("cc", gs, 0))


def test_loop_trips_are_global():
    """etg_stats.iterations of a communicator handle counts the loop trips, the
    same on every rank: BFS along a directed path of L vertices takes L - 1."""
    L = 200
    off = torch.zeros(L + 1, dtype=torch.int64)
    off[1:L] = torch.arange(1, L)
    off[L:] = L - 1
    col = torch.arange(1, L, dtype=torch.int64)
    parts = edist.local_partitions(off, col, None, L, 3)
    sts = edist._in_threads([lambda p=p: p.run(etg.BFS, 0)[1].iterations for p in parts])
    assert sts == [L - 1] * 3
