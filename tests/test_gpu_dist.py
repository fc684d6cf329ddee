"""The partitioned (multi-GPU) path with the CUDA engine, P partitions on one
GPU driven in lockstep by the same driver the NCCL ranks use (LoopbackGroup):
the assembled labels must equal the oracle's bit for bit."""
import numpy as np
import pytest
import torch

import graphgen as gg
import oracle

pytestmark = pytest.mark.gpu
etg = pytest.importorskip("paper_conf_ipps_wangzlg19_b200")
from paper_conf_ipps_wangzlg19_b200 import dist as edist  # noqa: E402

ALG = {"bfs": etg.BFS, "sssp": etg.SSSP, "cc": etg.CC, "sswp": etg.SSWP}


def engines(g, P, K=32, flags=0, sssp_delta=0):
    bounds = edist.partition_ranges(g.off, g.col, g.n, P)
    out = []
    for r in range(P):
        loff, lcol, lw = edist.partition_csr(g.off, g.col, g.w, g.n, bounds[r], bounds[r + 1])
        o, c, w, fl = etg.csr_to_device(loff, lcol, lw, device="cuda")
        G = etg.Graph(o, c, w, n=g.n, K=K, flags=flags | fl, symmetric=g.symmetric, sssp_delta=sssp_delta)
        out.append(edist.CudaEngine(G))
    return out


def expected(alg, g, s):
    off, col, w = g.numpy()
    return {"bfs": lambda: oracle.bfs(off, col, s), "sssp": lambda: oracle.sssp(off, col, w, s),
            "sswp": lambda: oracle.sswp(off, col, w, s), "cc": lambda: oracle.cc(off, col)}[alg]()


@pytest.mark.parametrize("alg", ["bfs", "sssp", "cc", "sswp"])
@pytest.mark.parametrize("P", [2, 3, 4])
def test_partitioned_c1(alg, P):
    g = gg.make("C1", symmetric=(alg == "cc"), weights=(alg != "cc"))
    s = gg.sample_sources(g, 1, P)[0]
    labels, st = edist.run_partitions(engines(g, P), edist.LoopbackGroup(), ALG[alg], s)
    np.testing.assert_array_equal(etg.to_u32_numpy(labels), expected(alg, g, s))


def test_partitioned_bfs_work_is_split():
    """Every edge of the activatable subgraph is relaxed on exactly one rank."""
    g = gg.make("T14", weights=False)
    s = gg.first_source(g)
    labels, st = edist.run_partitions(engines(g, 4), edist.LoopbackGroup(), etg.BFS, s)
    exp = expected("bfs", g, s)
    deg = np.diff(g.off.numpy())
    assert st.edges_processed == int(deg[exp != etg.INF].sum())
    np.testing.assert_array_equal(etg.to_u32_numpy(labels), exp)


def test_partitioned_k_and_flags():
    g = gg.make("LJ-small")
    s = gg.sample_sources(g, 1, 9)[0]
    for K, flags in ((8, 0), (1024, 0), (32, etg.NO_UDC)):
        labels, _ = edist.run_partitions(engines(g, 3, K, flags), edist.LoopbackGroup(), etg.SSSP, s)
        np.testing.assert_array_equal(etg.to_u32_numpy(labels), expected("sssp", g, s))


@pytest.mark.parametrize("P", [1, 2, 3])
@pytest.mark.parametrize("delta", [1, 16, 1 << 20])
def test_partitioned_near_far_sssp(P, delta):
    """The near-far SSSP schedule through the step-wise API: deferred vertices keep a
    stale snapshot (identical on every rank after the label exchange), an empty
    near set re-scans with the next threshold."""
    g = gg.make("C1")
    s = gg.sample_sources(g, 1, 77 + P)[0]
    labels, st = edist.run_partitions(engines(g, P, sssp_delta=delta), edist.LoopbackGroup(), etg.SSSP, s)
    np.testing.assert_array_equal(etg.to_u32_numpy(labels), expected("sssp", g, s))


# --------------------------------------------------------------------------- #
# NEXT-3: source partition + push exchange (etg_push_count/pack/apply)
# --------------------------------------------------------------------------- #
def src_engines(g, P, K=32, flags=0):
    bounds = edist.partition_ranges(g.off, g.col, g.n, P, by="out")
    out = []
    for r in range(P):
        loff, lcol, lw = edist.partition_csr_src(g.off, g.col, g.w, g.n, bounds[r], bounds[r + 1])
        o, c, w, fl = etg.csr_to_device(loff, lcol, lw, device="cuda")
        G = etg.Graph(o, c, w, n=g.n, K=K, flags=flags | fl, symmetric=g.symmetric)
        out.append(edist.CudaEngine(G))
    return bounds, out


def owned_labels(engs, bounds):
    return np.concatenate([etg.to_u32_numpy(e.labels)[bounds[r]:bounds[r + 1]] for r, e in enumerate(engs)])


@pytest.mark.parametrize("mode", ["sparse", "dense", "auto"])
@pytest.mark.parametrize("alg", ["sssp", "cc", "sswp"])
@pytest.mark.parametrize("P", [2, 3, 4])
def test_push_c1(alg, P, mode):
    g = gg.make("C1", symmetric=(alg == "cc"), weights=(alg != "cc"))
    s = gg.sample_sources(g, 1, 11 + P)[0]
    bounds, engs = src_engines(g, P)
    _, st, used = edist.run_push(engs, edist.LoopbackGroup(), ALG[alg], s, bounds, list(range(P)), mode)
    np.testing.assert_array_equal(owned_labels(engs, bounds), expected(alg, g, s))
    if mode != "auto":
        assert used[mode] == sum(used.values()) > 0


def test_push_lj_small_k_and_udc_off():
    g = gg.make("LJ-small")
    s = gg.sample_sources(g, 1, 5)[0]
    for K, flags in ((32, 0), (8, 0), (32, etg.NO_UDC)):
        bounds, engs = src_engines(g, 3, K, flags)
        edist.run_push(engs, edist.LoopbackGroup(), etg.SSSP, s, bounds, [0, 1, 2])
        np.testing.assert_array_equal(owned_labels(engs, bounds), expected("sssp", g, s))


def test_push_pack_pairs_are_the_moved_foreign_labels():
    """After one expand from the source: the packed pairs are exactly the
    vertices outside the owned range whose label the expand lowered, each once,
    grouped by owner, with the label value."""
    g = gg.make("C1")
    s = gg.first_source(g)
    P = 3
    bounds, engs = src_engines(g, P)
    r = next(q for q in range(P) if bounds[q] <= s < bounds[q + 1])
    e = engs[r]
    e.begin(etg.SSSP, s)
    e.expand()
    lab = etg.to_u32_numpy(e.labels).copy()
    off, col, w = g.numpy()
    nb = col[off[s]:off[s + 1]]
    foreign = sorted(set(int(u) for u in nb if not (bounds[r] <= u < bounds[r + 1])))
    counts = e.push_count(bounds, r)
    assert counts[r] == 0 and sum(counts) == len(foreign)
    pairs = e.push_pack(counts, r).cpu().numpy().view(np.uint32)
    start = 0
    for q in range(P):
        seg = pairs[start:start + counts[q]]
        assert all(bounds[q] <= u < bounds[q + 1] for u in seg[:, 0])
        start += counts[q]
    assert sorted(pairs[:, 0].tolist()) == foreign
    assert all(lab[u] == val for u, val in pairs)
    assert sum(e.push_count(bounds, r)) == 0            # packed = sent: snapshot refreshed
    e.end()


# --------------------------------------------------------------------------- #
# fused push exchange over peer memory (etg_push_peers): the expand kernel
# writes the owners' label arrays itself
# --------------------------------------------------------------------------- #
@pytest.mark.parametrize("alg", ["sssp", "cc", "sswp"])
@pytest.mark.parametrize("P", [2, 3, 4])
def test_push_p2p_c1(alg, P):
    g = gg.make("C1", symmetric=(alg == "cc"), weights=(alg != "cc"))
    s = gg.sample_sources(g, 1, 31 + P)[0]
    bounds, engs = src_engines(g, P)
    for r, e in enumerate(engs):
        e.set_peers(bounds, r, [x.labels.data_ptr() for x in engs])
    _, st, used = edist.run_push(engs, edist.LoopbackGroup(), ALG[alg], s, bounds, list(range(P)), "p2p")
    np.testing.assert_array_equal(owned_labels(engs, bounds), expected(alg, g, s))
    assert used["p2p"] > 0 and used["sparse"] == used["dense"] == 0


def test_push_peers_rejects_bad_arguments():
    g = gg.make("C1")
    bounds, engs = src_engines(g, 2)
    e = engs[0]
    ptrs = [x.labels.data_ptr() for x in engs]
    for bad in ([0, 5, 7], ):                        # bounds not ending at n
        with pytest.raises(etg.EtgError):
            e.set_peers(bad, 0, ptrs)
    with pytest.raises(etg.EtgError):
        e.set_peers(bounds, 2, ptrs)                  # rank >= P
    with pytest.raises(etg.EtgError):
        e.set_peers([0] + [g.n] * 9, 0, [ptrs[0]] * 9)  # P = 9 > 8


def _ipc_worker(rank, world, port, alg, out):
    import os
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    g = gg.make("C1", symmetric=(alg == "cc"), weights=(alg != "cc"))
    s = gg.first_source(g)
    dg = edist.PushDistGraph(g.off, g.col, g.w, g.n, rank, world, symmetric=g.symmetric,
                             device="cuda", mode="p2p")
    labels, st = dg.run(ALG[alg], s)
    lo, hi = dg.bounds[rank], dg.bounds[rank + 1]
    np.save(out + f".{rank}.npy", etg.to_u32_numpy(labels)[lo:hi])
    dist.barrier()
    dg.close()
    dist.destroy_process_group()


@pytest.mark.parametrize("alg", ["sssp", "cc"])
def test_push_p2p_two_processes_cuda_ipc(alg, tmp_path):
    """Two processes (two ranks) sharing the GPU: each maps the other's label
    array with CUDA IPC (etg_ipc_handle/open) and its expand kernel reduces
    into it directly -- the multi-GPU plumbing, with gloo for the host barrier."""
    import os
    import torch.multiprocessing as mp
    port = 32500 + (os.getpid() % 1000) + ALG[alg]
    out = str(tmp_path / "lab")
    mp.spawn(_ipc_worker, args=(2, port, alg, out), nprocs=2, join=True)
    g = gg.make("C1", symmetric=(alg == "cc"), weights=(alg != "cc"))
    got = np.concatenate([np.load(out + f".{r}.npy") for r in range(2)])
    np.testing.assert_array_equal(got, expected(alg, g, gg.first_source(g)))


# --------------------------------------------------------------------------- #
# fused destination-partition exchange (etg_dest_peers / etg_step_publish):
# owners store their changes straight into the peers' copies, no collective
# --------------------------------------------------------------------------- #
@pytest.mark.parametrize("alg", ["bfs", "sssp", "cc", "sswp"])
@pytest.mark.parametrize("P", [2, 3, 4])
def test_dest_p2p_c1(alg, P):
    g = gg.make("C1", symmetric=(alg == "cc"), weights=(alg != "cc"))
    s = gg.sample_sources(g, 1, 51 + P)[0]
    engs = engines(g, P)
    bounds = edist.partition_ranges(g.off, g.col, g.n, P)
    for r, e in enumerate(engs):
        e.set_dest_peers(bounds, r, [x.q.data_ptr() for x in engs], [x.labels.data_ptr() for x in engs])
    labels, st = edist.run_partitions(engs, edist.LoopbackGroup(), ALG[alg], s, bounds, "p2p")
    exp = expected(alg, g, s)
    for e in engs:
        np.testing.assert_array_equal(etg.to_u32_numpy(e.labels), exp)


def test_dest_p2p_near_far_sssp():
    g = gg.make("C1")
    s = gg.sample_sources(g, 1, 5)[0]
    P = 3
    engs = engines(g, P, sssp_delta=16)
    bounds = edist.partition_ranges(g.off, g.col, g.n, P)
    for r, e in enumerate(engs):
        e.set_dest_peers(bounds, r, [x.q.data_ptr() for x in engs], [x.labels.data_ptr() for x in engs])
    labels, _ = edist.run_partitions(engs, edist.LoopbackGroup(), etg.SSSP, s, bounds, "p2p")
    np.testing.assert_array_equal(etg.to_u32_numpy(labels), expected("sssp", g, s))


def _ipc_dest_worker(rank, world, port, alg, out):
    import os
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    g = gg.make("C1", symmetric=(alg == "cc"), weights=(alg != "cc"))
    s = gg.first_source(g)
    dg = edist.DistGraph(g.off, g.col, g.w, g.n, rank, world, symmetric=g.symmetric, device="cuda",
                         exchange="p2p")
    labels, st = dg.run(ALG[alg], s)
    np.save(out + f".{rank}.npy", etg.to_u32_numpy(labels))
    dist.barrier()
    dg.close()
    dist.destroy_process_group()


@pytest.mark.parametrize("alg", ["bfs", "sssp"])
def test_dest_p2p_two_processes_cuda_ipc(alg, tmp_path):
    """Two ranks in two processes sharing the GPU: each maps the other's bitmap
    and label array over CUDA IPC and publishes its owned changes into them."""
    import os
    import torch.multiprocessing as mp
    port = 33500 + (os.getpid() % 1000) + ALG[alg]
    out = str(tmp_path / "lab")
    mp.spawn(_ipc_dest_worker, args=(2, port, alg, out), nprocs=2, join=True)
    g = gg.make("C1", symmetric=(alg == "cc"), weights=(alg != "cc"))
    exp = expected(alg, g, gg.first_source(g))
    for r in range(2):
        np.testing.assert_array_equal(np.load(out + f".{r}.npy"), exp)


def test_exchange_entry_points_reject_misuse():
    """Error paths of the NEXT-3 / peer-memory entry points (ETG_EINVAL, no crash)."""
    g = gg.make("C1")
    bounds, engs = src_engines(g, 2)
    e = engs[0]
    # push entries outside an SSSP/CC/SSWP step-wise run
    with pytest.raises(etg.EtgError):
        e.push_count(bounds, 0)
    e.begin(etg.BFS, gg.first_source(g))
    with pytest.raises(etg.EtgError):
        e.push_count(bounds, 0)                       # BFS keeps the destination partition
    with pytest.raises(etg.EtgError):
        e.publish()                                   # no etg_dest_peers
    e.end()
    qp = [x.q.data_ptr() for x in engs]
    lp = [x.labels.data_ptr() for x in engs]
    with pytest.raises(etg.EtgError):
        e.set_dest_peers([0, 33, g.n], 0, qp, lp)     # inner bound not a multiple of 32
    with pytest.raises(etg.EtgError):
        e.set_dest_peers([0, 64, g.n], 2, qp, lp)     # rank >= P
    with pytest.raises(etg.EtgError):
        e.set_dest_peers([0, 64, g.n - 1], 0, qp, lp) # bounds must end at n
