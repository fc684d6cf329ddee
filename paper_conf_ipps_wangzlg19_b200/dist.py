"""Multi-GPU partitions: host-side partitioning + communicator bootstrap.

Design:

* vertex range R_g = [lo_g, hi_g) per rank, boundaries multiples of 32 (one
  bitmap word has one owner), chosen so every rank owns about the same number
  of IN-edges (destination partition: the work of a push relaxation lands on
  the destination) or OUT-edges (source partition, ``exchange="push"``);
* destination partition: rank g holds E_g = {(u, v) in E : v in R_g} as a CSR
  over all n sources (global ids), so its relaxations only touch owned
  vertices; source partition: rank g holds the out-edges of R_g.

Everything after the partitioning runs inside libetg.so: ``Graph(...,
comm=...)`` maps the peers' workspaces (etg_load_csr on a communicator) and
every traversal call runs the whole partitioned Proc. 1 loop -- expand,
exchange over peer memory, barrier, scan, termination count -- in C++ and the
library's kernels.  This module holds no exchange arithmetic: torch.distributed
is used once, to hand rank 0's communicator id to the other ranks.
"""
from __future__ import annotations

import threading
from typing import List, Optional, Sequence

import torch

from . import PUSH, Comm, EtgError, Graph, Stats, csr_to_device


# --------------------------------------------------------------------------- #
# partitioning (host logic; torch ops on whatever device the CSR lives on)
# --------------------------------------------------------------------------- #
def partition_ranges(off: torch.Tensor, col: torch.Tensor, n: int, P: int, align: int = 32,
                     by: str = "in") -> List[int]:
    """Boundaries lo_0 = 0 < ... < lo_P = n, multiples of `align` (except n),
    balancing in-edge counts (by="in": destination partition) or out-edge
    counts (by="out": source partition, the push exchange).  Returns the P + 1
    boundaries."""
    if P < 1:
        raise ValueError("P >= 1")
    if by == "out":
        deg = (off[1:].to(torch.int64) - off[:-1].to(torch.int64))
    else:
        deg = torch.bincount(col.to(torch.int64), minlength=n)
    cum = torch.cumsum(deg, 0)
    m = int(cum[-1]) if n else 0
    bounds = [0]
    for g in range(1, P):
        target = (m * g) // P
        v = int(torch.searchsorted(cum, torch.tensor(target, device=cum.device)))
        v = (v + align // 2) // align * align
        v = min(max(v, bounds[-1]), n)
        bounds.append(v)
    bounds.append(n)
    return bounds


def partition_csr(off: torch.Tensor, col: torch.Tensor, w: Optional[torch.Tensor], n: int,
                  lo: int, hi: int, chunk: int = 1 << 28):
    """The rank's destination-partitioned CSR: rows = all n sources, edges with
    destination in [lo, hi), CSR order kept, global ids.  Processed in edge
    chunks (no m-sized int64 temporaries), kept columns stored as int32 bits."""
    off = off.to(torch.int64)
    m = int(col.shape[0])
    dev = off.device
    cnt = torch.zeros(n, dtype=torch.int64, device=dev)
    cols, ws = [], []
    for a in range(0, m, chunk):
        b = min(m, a + chunk)
        c = col[a:b].to(torch.int64)
        keep = (c >= lo) & (c < hi)
        src = torch.searchsorted(off, torch.arange(a, b, device=dev), right=True) - 1
        cnt += torch.bincount(src[keep], minlength=n)
        cols.append(c[keep].to(torch.int32))
        if w is not None:
            ws.append(w[a:b][keep].to(torch.int32))
        del c, keep, src
    loff = torch.zeros(n + 1, dtype=torch.int64, device=dev)
    loff[1:] = torch.cumsum(cnt, 0)
    lcol = torch.cat(cols) if cols else torch.zeros(0, dtype=torch.int32, device=dev)
    lw = (torch.cat(ws) if ws else torch.zeros(0, dtype=torch.int32, device=dev)) if w is not None else None
    return loff, lcol, lw


def partition_csr_src(off: torch.Tensor, col: torch.Tensor, w: Optional[torch.Tensor], n: int,
                      lo: int, hi: int):
    """The rank's SOURCE-partitioned CSR (push exchange, NEXT-3): rows = all n
    sources, only the rows of [lo, hi) keep their out-edges (global ids)."""
    off = off.to(torch.int64)
    a, b = int(off[lo]), int(off[hi])
    loff = (off.clamp(min=a, max=b) - a)
    loff[:lo] = 0
    loff[hi:] = b - a
    lcol = col[a:b].to(torch.int32)
    lw = None if w is None else w[a:b].to(torch.int32)
    return loff, lcol, lw


# --------------------------------------------------------------------------- #
# bootstrap
# --------------------------------------------------------------------------- #
def comm_from_group(rank: int, world: int, device: int = -1, group=None) -> Comm:
    """Rank 0 makes the communicator id, torch.distributed hands it to the
    other ranks (broadcast_object_list on any backend, gloo included), every
    rank joins (etg_comm_init).  The only use of torch.distributed here."""
    obj = [Comm.unique_id() if rank == 0 else None]
    if world > 1:
        import torch.distributed as dist
        dist.broadcast_object_list(obj, src=0, group=group)
    return Comm(rank, world, obj[0], device)


class DistGraph:
    """This rank's partition of a graph over a :class:`Comm` (collective).

    exchange="dest": destination partition (every algorithm); "push": source
    partition with the fused push exchange (SSSP/CC/SSWP).  ``run`` returns
    this rank's owned slice of the labels and the statistics (summed over the
    ranks; ``ms`` = max over ranks)."""

    def __init__(self, off, col, w, n: int, comm: Comm, *, exchange: str = "dest", K: int = 32,
                 flags: int = 0, symmetric: bool = False, sssp_delta=0, device="cuda", bounds=None,
                 stream=None):
        if exchange not in ("dest", "push"):
            raise EtgError("exchange must be 'dest' or 'push'")
        rank, world = comm.rank, comm.world
        self.n, self.rank, self.world, self.exchange = n, rank, world, exchange
        by = "out" if exchange == "push" else "in"
        self.bounds = list(bounds) if bounds is not None else partition_ranges(off, col, n, world, by=by)
        lo, hi = self.bounds[rank], self.bounds[rank + 1]
        part = partition_csr_src if exchange == "push" else partition_csr
        loff, lcol, lw = part(off, col, w, n, lo, hi)
        o, c, ww, fl = csr_to_device(loff, lcol, lw, device=device)
        del loff, lcol, lw
        self.graph = Graph(o, c, ww, n=n, K=K, flags=flags | fl | (PUSH if exchange == "push" else 0),
                           symmetric=symmetric, sssp_delta=sssp_delta, comm=comm, v_lo=lo, v_hi=hi,
                           stream=stream)
        self.lo, self.hi = lo, hi

    def run(self, alg: int, source: int = 0, out: Optional[torch.Tensor] = None):
        return self.graph.run(alg, source, out)

    def close(self):
        self.graph.close()


# --------------------------------------------------------------------------- #
# P partitions inside ONE process (one thread and one CUDA stream per rank):
# the same library path as separate processes, peers reached by plain device
# pointers instead of CUDA IPC.  For tests and single-GPU experiments.
# --------------------------------------------------------------------------- #
def _in_threads(fns: Sequence):
    out, err = [None] * len(fns), []

    def body(i):
        try:
            out[i] = fns[i]()
        except BaseException as e:       # surfaced in the caller
            err.append(e)
    ts = [threading.Thread(target=body, args=(i,)) for i in range(len(fns))]
    for t in ts:
        t.start()
    for t in ts:
        t.join()
    if err:
        raise err[0]
    return out


def local_partitions(off, col, w, n: int, P: int, *, exchange: str = "dest", device="cuda",
                     **kw) -> List[DistGraph]:
    """P DistGraph ranks of one graph in this process, over one communicator."""
    uid = Comm.unique_id()
    dev = torch.device(device)
    di = dev.index if dev.index is not None else (torch.cuda.current_device() if dev.type == "cuda" else -1)
    by = "out" if exchange == "push" else "in"
    bounds = kw.pop("bounds", None) or partition_ranges(off, col, n, P, by=by)

    def make(r):
        def f():
            if dev.type == "cuda":
                torch.cuda.set_device(di)
            comm = Comm(r, P, uid, di)
            s = torch.cuda.Stream(device=dev)
            with torch.cuda.stream(s):
                return DistGraph(off, col, w, n, comm, exchange=exchange, device=dev, bounds=bounds,
                                 stream=s, **kw)
        return f
    return _in_threads([make(r) for r in range(P)])


def run_local(parts: Sequence[DistGraph], alg: int, source: int = 0):
    """One collective traversal of P in-process ranks: (the owned slices
    concatenated in rank order = the labels of all n vertices, rank 0's stats)."""
    def make(p):
        def f():
            with torch.cuda.stream(p.graph._stream):
                return p.run(alg, source)
        return f
    res = _in_threads([make(p) for p in parts])
    torch.cuda.synchronize()
    labels = torch.cat([lab[:p.hi - p.lo] for p, (lab, _) in zip(parts, res)])
    return labels, res[0][1]
