"""Multi-rank host logic on the CPU (no GPU needed).

* partition properties (every edge in exactly one part, word-aligned ranges,
  in-/out-edge balance);
* the library's communicator (etg_comm_*: shared-memory rendezvous and host
  barrier, include/etg.h), which is the control plane of the partitioned loop:
  P threads in one process, world_size 2 over gloo (torch.distributed only
  hands rank 0's id to rank 1, 127.0.0.1), argument errors, a missing peer
  (timeout) and a dead peer, each reported as an error instead of a hang.
The partitioned traversal itself (C++ loop + peer-memory kernels) is covered
on the GPU by tests/test_gpu_dist.py.
"""
import os
import threading
import time

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import graphgen as gg
import paper_conf_ipps_wangzlg19_b200 as etg
from paper_conf_ipps_wangzlg19_b200 import _build
from paper_conf_ipps_wangzlg19_b200 import dist as edist


@pytest.fixture(scope="module", autouse=True)
def _lib():
    _build.build()
    etg.lib()


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


@pytest.mark.parametrize("P", [1, 2, 3, 4])
def test_source_partition_properties(P):
    g = gg.make("T12")
    bounds = edist.partition_ranges(g.off, g.col, g.n, P, by="out")
    assert bounds[0] == 0 and bounds[-1] == g.n and all(b % 32 == 0 for b in bounds[:-1])
    deg = np.diff(g.off.numpy())
    tot = 0
    for r in range(P):
        lo, hi = bounds[r], bounds[r + 1]
        loff, lcol, lw = edist.partition_csr_src(g.off, g.col, g.w, g.n, lo, hi)
        ldeg = np.diff(loff.numpy())
        assert np.array_equal(ldeg[lo:hi], deg[lo:hi]) and ldeg[:lo].sum() == 0 and ldeg[hi:].sum() == 0
        a = int(g.off[lo])
        assert torch.equal(lcol, g.col[a:a + lcol.shape[0]].to(torch.int32))
        assert abs(deg[lo:hi].sum() / g.m - 1 / P) < 0.05
        tot += lcol.shape[0]
    assert tot == g.m


# --------------------------------------------------------------------------- #
# communicator
# --------------------------------------------------------------------------- #
def test_comm_barrier_threads():
    """P ranks as threads: after barrier k every rank sees all P arrivals of phase k."""
    P, rounds = 4, 200
    uid = etg.Comm.unique_id()
    assert len(uid) == 128 and uid != etg.Comm.unique_id()
    arrivals = [0] * rounds
    lock = threading.Lock()
    bad = []

    def rank(r):
        c = etg.Comm(r, P, uid)
        for k in range(rounds):
            with lock:
                arrivals[k] += 1
            c.barrier()
            if arrivals[k] != P:
                bad.append((r, k, arrivals[k]))
        c.close()
    ts = [threading.Thread(target=rank, args=(r,)) for r in range(P)]
    for t in ts:
        t.start()
    for t in ts:
        t.join()
    assert not bad and arrivals == [P] * rounds


def test_comm_argument_errors():
    uid = etg.Comm.unique_id()
    with pytest.raises(etg.EtgError, match="EINVAL"):
        etg.Comm(2, 2, uid)                               # rank >= world
    with pytest.raises(etg.EtgError, match="EINVAL"):
        etg.Comm(0, 9, uid)                               # world > 8
    with pytest.raises(etg.EtgError, match="EINVAL"):
        etg.Comm(0, 1, bytes(128))                        # not a unique id
    c = etg.Comm(0, 1, etg.Comm.unique_id())              # world 1: nothing to wait for
    c.barrier()
    c.close()


def test_comm_missing_peer_times_out(monkeypatch):
    monkeypatch.setenv("ETG_COMM_TIMEOUT_S", "1")
    t = time.time()
    with pytest.raises(etg.EtgError, match="ENCCL"):
        etg.Comm(0, 2, etg.Comm.unique_id())              # rank 1 never comes
    assert time.time() - t < 30


def _gloo_worker(rank, world, port, tmp, die):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    c = edist.comm_from_group(rank, world)
    for k in range(50):
        open(os.path.join(tmp, f"r{rank}.{k}"), "w").close()
        c.barrier()
        for q in range(world):                            # every rank's phase-k mark is there
            assert os.path.exists(os.path.join(tmp, f"r{q}.{k}"))
    if die and rank == 1:
        os._exit(0)                                       # leave without the next barrier
    if die:
        os.environ["ETG_COMM_TIMEOUT_S"] = "120"
        t = time.time()
        try:
            c.barrier()
            raise SystemExit(3)
        except etg.EtgError as e:
            assert "ENCCL" in str(e) and time.time() - t < 60
    else:
        c.barrier()
    c.close()
    open(os.path.join(tmp, f"ok{rank}"), "w").close()


@pytest.mark.parametrize("die", [False, True])
def test_comm_gloo_world2(tmp_path, die):
    """world_size 2 over gloo: the id travels by torch.distributed, the barrier
    orders the ranks; a rank that dies is detected (ENCCL), not waited for."""
    port = 29600 + os.getpid() % 200 + (7 if die else 0)
    mp.spawn(_gloo_worker, args=(2, port, str(tmp_path), die), nprocs=2, join=True)
    assert os.path.exists(tmp_path / "ok0")
    assert die or os.path.exists(tmp_path / "ok1")
