"""Multi-GPU traversal: 1-D destination-range partition + per-iteration exchange.

Design:

* vertex range R_g = [lo_g, hi_g) per rank, boundaries multiples of 32 (one
  bitmap word has one owner), chosen so every rank owns about the same number
  of IN-edges (the work of a push relaxation lands on the destination);
* rank g holds E_g = {(u, v) in E : v in R_g} as a CSR over all n sources
  (global ids) -- relaxations on rank g only ever touch owned vertices;
* every rank expands the same, replicated, compacted active set (UDC over its
  own sub-rows, so a hub's edges are split ~deg/P per rank), marks improved
  owned vertices in its bitmap (BFS, near-far SSSP), then the exchange makes
  the bitmaps the union and, for SSSP/CC/SSWP, the labels the element-wise best
  (MIN; MAX for SSWP): a non-owner's copy is the owner's value from an earlier
  exchange, never better than the owner's current one.  Union = unsigned MAX
  per word: a word's new bits come from its owner only, and the bits every
  rank holds already (near-far's deferred vertices) are the same on all ranks,
  so the owner's word is a superset of every other rank's.  SSSP/CC/SSWP mark
  nothing otherwise: each rank's scan activates the vertices whose (exchanged)
  label moved.  BFS exchanges the bitmap only -- each rank's scan writes the
  depth of every vertex of the new active set.
* collective: an all-gather of the owned slices (bitmap words, labels) -- see
  ``_exchange``; a full-array all-reduce (MAX on the bitmap, MIN/MAX on the
  labels) is kept as the fallback without partition bounds;
* termination: the number of activated vertices (bitmap bits consumed by the
  scan) is identical on every rank after the exchange, so all ranks leave the
  loop together (the compacted sizes differ: they count local out-edges).

Only argument marshalling and the collective calls are in Python; every step of
the traversal runs in libetg.so (etg_step_begin / etg_step_expand /
etg_step_scan / etg_step_end).  The collective is torch.distributed (NCCL over
NVLink on the GPU box); ``LoopbackGroup`` runs P partitions on one GPU for
tests.
"""
from __future__ import annotations

import ctypes
from typing import Callable, List, Optional, Sequence

import torch

from . import (BFS, CC, SSSP, SSWP, EtgError, Graph, Stats, _check, _ptr, lib)

SIGN = -(1 << 31)   # xor with this maps uint32 order onto int32 order


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
# collectives
# --------------------------------------------------------------------------- #
class TorchDistGroup:
    """Collectives over a torch.distributed process group (NCCL on GPUs, gloo on CPUs)."""

    def __init__(self, group=None):
        import torch.distributed as dist
        self.dist = dist
        self.group = group

    def allreduce(self, tensors: Sequence[torch.Tensor], op: str) -> None:
        ops = {"sum": self.dist.ReduceOp.SUM, "min": self.dist.ReduceOp.MIN,
               "max": self.dist.ReduceOp.MAX}
        assert len(tensors) == 1
        self.dist.all_reduce(tensors[0], op=ops[op], group=self.group)

    def allgather_ranges(self, tensors: Sequence[torch.Tensor], bounds: Sequence[int]) -> None:
        """Rank r's slice [bounds[r], bounds[r+1]) of its tensor is authoritative:
        after the call every rank's tensor holds every rank's slice (one
        all-gather of equal-sized, padded slices)."""
        assert len(tensors) == 1
        t = tensors[0]
        r = self.dist.get_rank(self.group)
        P = len(bounds) - 1
        width = max(bounds[q + 1] - bounds[q] for q in range(P))
        send = torch.zeros(width, dtype=t.dtype, device=t.device)
        send[:bounds[r + 1] - bounds[r]] = t[bounds[r]:bounds[r + 1]]
        recv = [torch.empty_like(send) for _ in range(P)]
        self.dist.all_gather(recv, send, group=self.group)
        for q in range(P):
            if q != r:
                t[bounds[q]:bounds[q + 1]] = recv[q][:bounds[q + 1] - bounds[q]]


    def barrier(self) -> None:
        self.dist.barrier(group=self.group)

    def alltoallv(self, sends: Sequence[torch.Tensor], counts: Sequence[Sequence[int]]) -> List[torch.Tensor]:
        """sends[0]: this rank's rows (int32 [k, 2]) grouped by destination rank,
        counts[0][q] rows for rank q.  Returns [rows received, grouped by source]."""
        assert len(sends) == 1
        send, cnt = sends[0], list(counts[0])
        P = len(cnt)
        c = torch.tensor(cnt, dtype=torch.int64, device=send.device)
        rc = torch.empty_like(c)
        self.dist.all_to_all_single(rc, c, group=self.group)
        rcnt = [int(x) for x in rc.cpu()]
        recv = torch.empty((sum(rcnt), send.shape[1]), dtype=send.dtype, device=send.device)
        if P and (sum(rcnt) or sum(cnt)):
            self.dist.all_to_all_single(recv, send, output_split_sizes=rcnt, input_split_sizes=cnt,
                                        group=self.group)
        return [recv]

    def reduce_ranges(self, tensors: Sequence[torch.Tensor], bounds: Sequence[int], op: str) -> None:
        """Rank r's slice [bounds[r], bounds[r+1]) becomes the element-wise `op`
        (min/max, int32 order) over all ranks' tensors; other slices are left
        as they are.  NCCL: one reduce-scatter of padded slices; gloo (no
        reduce-scatter): an all-reduce of the whole tensor."""
        assert len(tensors) == 1
        t = tensors[0]
        r = self.dist.get_rank(self.group)
        P = len(bounds) - 1
        ops = {"min": self.dist.ReduceOp.MIN, "max": self.dist.ReduceOp.MAX}
        if self.dist.get_backend(self.group) != "nccl":
            acc = t.clone()
            self.dist.all_reduce(acc, op=ops[op], group=self.group)
            t[bounds[r]:bounds[r + 1]] = acc[bounds[r]:bounds[r + 1]]
            return
        width = max(bounds[q + 1] - bounds[q] for q in range(P))
        pad = 0x7FFFFFFF if op == "min" else -(1 << 31)
        inp = torch.full((P, width), pad, dtype=t.dtype, device=t.device)
        for q in range(P):
            inp[q, :bounds[q + 1] - bounds[q]] = t[bounds[q]:bounds[q + 1]]
        out = torch.empty(width, dtype=t.dtype, device=t.device)
        self.dist.reduce_scatter_tensor(out, inp.reshape(-1), op=ops[op], group=self.group)
        t[bounds[r]:bounds[r + 1]] = out[:bounds[r + 1] - bounds[r]]


class LoopbackGroup:
    """P 'ranks' in one process (one GPU): all_reduce over a list of tensors."""

    def allreduce(self, tensors: Sequence[torch.Tensor], op: str) -> None:
        acc = tensors[0].clone()
        for t in tensors[1:]:
            if op == "sum":
                acc += t
            elif op == "min":
                acc = torch.minimum(acc, t)
            else:
                acc = torch.maximum(acc, t)
        for t in tensors:
            t.copy_(acc)

    def allgather_ranges(self, tensors: Sequence[torch.Tensor], bounds: Sequence[int]) -> None:
        for q, src in enumerate(tensors):
            for t in tensors:
                if t is not src:
                    t[bounds[q]:bounds[q + 1]] = src[bounds[q]:bounds[q + 1]]


    def barrier(self) -> None:
        pass

    def alltoallv(self, sends: Sequence[torch.Tensor], counts: Sequence[Sequence[int]]) -> List[torch.Tensor]:
        P = len(sends)
        starts = [[sum(counts[q][:r]) for r in range(P)] for q in range(P)]
        return [torch.cat([sends[q][starts[q][r]:starts[q][r] + counts[q][r]] for q in range(P)])
                for r in range(P)]

    def reduce_ranges(self, tensors: Sequence[torch.Tensor], bounds: Sequence[int], op: str) -> None:
        for r, t in enumerate(tensors):
            lo, hi = bounds[r], bounds[r + 1]
            acc = t[lo:hi].clone()
            for o in tensors:
                acc = torch.minimum(acc, o[lo:hi]) if op == "min" else torch.maximum(acc, o[lo:hi])
            t[lo:hi] = acc


# --------------------------------------------------------------------------- #
# engines: the CUDA handle (product) behind a small step interface
# --------------------------------------------------------------------------- #
class CudaEngine:
    """One partition on one GPU, driven step-wise through the C ABI."""

    def __init__(self, graph: Graph):
        self.g = graph
        off = ctypes.c_size_t()
        nw = ctypes.c_uint32()
        _check(lib().etg_bitmap_layout(graph._h, ctypes.byref(off), ctypes.byref(nw)), "etg_bitmap_layout")
        self.q = graph.workspace[off.value: off.value + 4 * nw.value].view(torch.int32)
        self.labels = torch.empty(graph.n, dtype=torch.int32, device=graph.device)

    def begin(self, alg: int, source: int) -> int:
        na = ctypes.c_uint32()
        _check(lib().etg_step_begin(self.g._h, alg, source, _ptr(self.labels), ctypes.byref(na)),
               "etg_step_begin")
        return int(na.value)

    def expand(self) -> None:
        _check(lib().etg_step_expand(self.g._h), "etg_step_expand")

    def scan(self) -> int:
        na = ctypes.c_uint32()
        _check(lib().etg_step_scan(self.g._h, ctypes.byref(na)), "etg_step_scan")
        return int(na.value)

    def end(self) -> Stats:
        st = Stats()
        _check(lib().etg_step_end(self.g._h, ctypes.byref(st)), "etg_step_end")
        return st

    # ---- push exchange (source partition, NEXT-3) ----
    def frontier(self) -> int:
        """Compacted active-set size of the last scan (vertices with local out-edges)."""
        out = (ctypes.c_uint64 * 6)()
        _check(lib().etg_debug_counters(self.g._h, out), "etg_debug_counters")
        return int(out[1])

    def push_count(self, bounds: Sequence[int], rank: int) -> List[int]:
        P = len(bounds) - 1
        self._bounds = torch.tensor(list(bounds), dtype=torch.int64).to(torch.int32).to(self.labels.device)
        self._counts = torch.zeros(P, dtype=torch.int64, device=self.labels.device)
        _check(lib().etg_push_count(self.g._h, P, rank, _ptr(self._bounds), _ptr(self._counts)), "etg_push_count")
        return [int(x) for x in self._counts.cpu()]

    def push_pack(self, counts: Sequence[int], rank: int) -> torch.Tensor:
        P = len(counts)
        cur = torch.tensor([sum(counts[:q]) for q in range(P)], dtype=torch.int64, device=self.labels.device)
        pairs = torch.empty((max(sum(counts), 1), 2), dtype=torch.int32, device=self.labels.device)
        _check(lib().etg_push_pack(self.g._h, P, rank, _ptr(self._bounds), _ptr(cur), _ptr(pairs)), "etg_push_pack")
        return pairs[:sum(counts)]

    def set_peers(self, bounds: Sequence[int], rank: int, peer_ptrs: Sequence[int]) -> None:
        """Fused push exchange: relaxations of vertices owned by rank q also land
        in peer_ptrs[q] (rank q's label array, mapped into this process)."""
        P = len(bounds) - 1
        b = (ctypes.c_uint32 * (P + 1))(*bounds)
        ptrs = (ctypes.c_void_p * P)(*peer_ptrs)
        _check(lib().etg_push_peers(self.g._h, P, rank, b, ptrs), "etg_push_peers")
        self.peered = P > 1

    def sync(self) -> None:
        torch.cuda.synchronize(self.labels.device)

    # ---- fused destination-partition exchange ----
    def set_dest_peers(self, bounds: Sequence[int], rank: int, q_ptrs: Sequence[int],
                       label_ptrs: Sequence[int]) -> None:
        """etg_step_publish will store this rank's changes straight into the peers' copies."""
        P = len(bounds) - 1
        b = (ctypes.c_uint32 * (P + 1))(*bounds)
        qp = (ctypes.c_void_p * P)(*q_ptrs)
        lp = (ctypes.c_void_p * P)(*label_ptrs)
        _check(lib().etg_dest_peers(self.g._h, P, rank, b, qp, lp), "etg_dest_peers")
        self.dest_peered = True

    def publish(self) -> None:
        _check(lib().etg_step_publish(self.g._h), "etg_step_publish")

    def push_apply(self, pairs: torch.Tensor) -> None:
        pairs = pairs.contiguous()
        _check(lib().etg_push_apply(self.g._h, _ptr(pairs), int(pairs.shape[0])), "etg_push_apply")


def _exchange(engines, group, alg: int, bounds: Optional[Sequence[int]] = None) -> None:
    """Union of the bitmaps; best labels (SSSP/CC: min, SSWP: max) -- see module doc.

    With the partition bounds: an all-gather of every rank's OWNED slices (its
    bitmap words and, for SSSP/CC/SSWP, its labels).  Relaxations only ever
    touch owned vertices, so the owner's slice already is the union / the
    best value, and each rank sends n/32 words / P (+ n labels / P) instead of
    reducing full-size arrays.  Without bounds: full-size all-reduces."""
    if bounds is not None:
        wb = [(b + 31) // 32 for b in bounds]          # boundaries are multiples of 32 (last: n)
        group.allgather_ranges([e.q for e in engines], wb)
        if alg != BFS:
            group.allgather_ranges([e.labels for e in engines], bounds)
        return
    qs = [e.q for e in engines]
    for t in qs:
        t.bitwise_xor_(SIGN)                # uint32 order -> int32 order
    group.allreduce(qs, "max")              # superset words: unsigned MAX = OR
    for t in qs:
        t.bitwise_xor_(SIGN)
    if alg != BFS:
        labs = [e.labels for e in engines]
        for t in labs:
            t.bitwise_xor_(SIGN)            # uint32 order -> int32 order
        group.allreduce(labs, "max" if alg == SSWP else "min")
        for t in labs:
            t.bitwise_xor_(SIGN)


def run_partitions(engines, group, alg: int, source: int = 0, bounds: Optional[Sequence[int]] = None,
                   exchange: str = "collective"):
    """Drive P engines in lockstep (all in this process: loopback), or ONE
    engine of this rank (torch.distributed: the other ranks run the same
    loop).  ``bounds`` (the partition, ``partition_ranges``) selects the
    all-gather exchange of owned slices; without it full arrays are
    all-reduced.  ``exchange="p2p"``: no collective -- each engine's
    etg_step_publish stores its owned changes straight into the peers' copies
    (engines set up with ``set_dest_peers``), then sync + barrier; barriers
    after the initialisation and after the scans keep a rank's stores out of a
    peer's copy until that peer has initialised it / finished scanning it.
    Returns (labels of engines[0], summed stats)."""
    if exchange == "p2p" and not all(getattr(e, "dest_peered", False) for e in engines):
        raise EtgError("exchange='p2p' needs set_dest_peers() on every engine")
    n_act = [e.begin(alg, source) for e in engines]
    if exchange == "p2p":
        group.barrier()     # every peer has initialised its copies before anyone publishes
    while n_act[0] > 0:
        for e in engines:
            e.expand()
        if exchange == "p2p":
            for e in engines:
                e.publish()
            for e in engines:
                e.sync()
            group.barrier()
        else:
            _exchange(engines, group, alg, bounds)
        n_act = [e.scan() for e in engines]
        if exchange == "p2p":
            # nobody publishes iteration k+1 into a peer still scanning iteration k
            group.barrier()
        if len(set(n_act)) != 1:
            raise EtgError(f"ranks disagree on the active-set size: {n_act}")
    stats = [e.end() for e in engines]
    total = Stats()
    total.iterations = stats[0].iterations
    for f in ("activations", "frontier_total", "shadows", "edges_processed"):
        setattr(total, f, sum(getattr(s, f) for s in stats))
    return engines[0].labels, total


def map_peer_tensors(t: torch.Tensor, rank: int, world: int, group=None):
    """CUDA IPC: every rank publishes the handle of its tensor t (all_gather_object)
    and maps every peer's into this process.  Returns (device pointers of the P
    ranks' tensors, valid in this process; mapped base addresses for etg_ipc_close)."""
    import torch.distributed as dist
    h = (ctypes.c_uint8 * 64)()
    off = ctypes.c_uint64()
    _check(lib().etg_ipc_handle(_ptr(t), h, ctypes.byref(off)), "etg_ipc_handle")
    allh = [None] * world
    dist.all_gather_object(allh, (bytes(h), int(off.value)), group=group)
    ptrs, bases = [], []
    for q, (hb, o) in enumerate(allh):
        if q == rank:
            ptrs.append(t.data_ptr())
            continue
        base = ctypes.c_void_p()
        _check(lib().etg_ipc_open((ctypes.c_uint8 * 64)(*hb), ctypes.byref(base)), "etg_ipc_open")
        bases.append(base.value)
        ptrs.append(base.value + o)
    return ptrs, bases


def open_peer_labels(engine: "CudaEngine", bounds: Sequence[int], rank: int, world: int, group=None) -> List[int]:
    """Push exchange over peer memory: map every peer's label array and register
    them with the engine (``set_peers``).  Returns the mapped bases."""
    ptrs, bases = map_peer_tensors(engine.labels, rank, world, group)
    engine.set_peers(bounds, rank, ptrs)
    return bases


def run_push(engines, group, alg: int, source: int, bounds: Sequence[int], ranks: Sequence[int],
             mode: str = "auto"):
    """NEXT-3: source partition + push exchange (SSSP/CC/SSWP).  Each engine
    holds the out-edges of its owned range (``partition_csr_src``) and expands
    only its own active vertices; labels it lowered on vertices it does not
    own are proposals for their owners.  Per iteration, after the expand:
      sparse -- (id, label) pairs of the moved non-owned vertices, grouped by
                owner, one all-to-all, then atomic min/max on the receiver;
      dense  -- element-wise min/max of the full label arrays onto each
                owner's range (reduce-scatter);
    ``mode="auto"`` picks whichever moves fewer bytes this iteration (8 bytes a
    pair against 4 (P - 1) n bytes dense); all ranks agree through one sum.
    ``mode="p2p"``: the fused exchange -- the expand kernel itself applies each
    relaxation of a foreign vertex to the owner's label array over peer memory
    (engines set up with ``set_peers``); the host only waits for every rank's
    expand (sync + barrier) before the scans.
    Stops when every rank's compacted active set is empty.  ``ranks``: the rank
    of each engine (all of 0..P-1 in loopback, [rank] under torch.distributed).
    Returns (labels of engines[0], summed stats, {"sparse": k, "dense": k})."""
    if alg == BFS:
        raise EtgError("the push exchange serves SSSP/CC/SSWP; BFS uses the destination partition")
    P = len(bounds) - 1
    n = bounds[-1]
    op = "max" if alg == SSWP else "min"
    used = {"sparse": 0, "dense": 0}
    for e in engines:
        e.begin(alg, source)

    def total(vals: List[int]) -> int:
        t = [torch.tensor([v], dtype=torch.int64, device=e.labels.device) for v, e in zip(vals, engines)]
        group.allreduce(t, "sum")
        return int(t[0].item())

    if mode == "p2p" and P > 1 and not all(getattr(e, "peered", False) for e in engines):
        raise EtgError("mode='p2p' needs set_peers() on every engine")
    while total([e.frontier() for e in engines]) > 0:
        for e in engines:
            e.expand()
        if mode == "p2p" and P > 1:
            used["p2p"] = used.get("p2p", 0) + 1
            for e in engines:
                e.sync()                            # this rank's remote reductions are done
            group.barrier()                         # ... and every other rank's
            for e in engines:
                e.scan()
            continue
        if P == 1:                                  # nothing is foreign
            for e in engines:
                e.scan()
            continue
        counts = [e.push_count(bounds, r) for e, r in zip(engines, ranks)]
        pairs = total([sum(c) for c in counts])
        sparse = mode == "sparse" or (mode == "auto" and 8 * pairs < 4 * (P - 1) * n)
        if sparse:
            used["sparse"] += 1
            sends = [e.push_pack(c, r) for e, c, r in zip(engines, counts, ranks)]
            recvs = group.alltoallv(sends, counts)
            for e, rv in zip(engines, recvs):
                e.push_apply(rv)
        else:
            used["dense"] += 1
            labs = [e.labels for e in engines]
            for t in labs:
                t.bitwise_xor_(SIGN)            # uint32 order -> int32 order
            group.reduce_ranges(labs, bounds, op)
            for t in labs:
                t.bitwise_xor_(SIGN)
        for e in engines:
            e.scan()
    stats = [e.end() for e in engines]
    tot = Stats()
    tot.iterations = stats[0].iterations
    for f in ("activations", "frontier_total", "shadows", "edges_processed"):
        setattr(tot, f, sum(getattr(s, f) for s in stats))
    return engines[0].labels, tot, used


class DistGraph:
    """This rank's partition of a graph, driven over a torch.distributed group.
    exchange="collective": all-gather of owned slices (NCCL); "p2p": each rank
    stores its owned changes straight into the peers' copies (CUDA IPC)."""

    def __init__(self, off, col, w, n: int, rank: int, world: int, *, K: int = 32, flags: int = 0,
                 symmetric: bool = False, device="cuda", group=None, bounds=None, exchange: str = "collective"):
        from . import csr_to_device
        self.n, self.rank, self.world = n, rank, world
        self.bounds = bounds if bounds is not None else partition_ranges(off, col, n, world)
        lo, hi = self.bounds[rank], self.bounds[rank + 1]
        loff, lcol, lw = partition_csr(off, col, w, n, lo, hi)
        o, c, ww, fl = csr_to_device(loff, lcol, lw, device=device)
        self.graph = Graph(o, c, ww, n=n, K=K, flags=flags | fl, symmetric=symmetric)
        self.engine = CudaEngine(self.graph)
        self.group = TorchDistGroup(group)
        self.exchange = exchange
        self._ipc = []
        if exchange == "p2p":
            if world > 1:
                qp, qb = map_peer_tensors(self.engine.q, rank, world, group)
                lp, lb = map_peer_tensors(self.engine.labels, rank, world, group)
                self._ipc = qb + lb
            else:
                qp, lp = [self.engine.q.data_ptr()], [self.engine.labels.data_ptr()]
            self.engine.set_dest_peers(self.bounds, rank, qp, lp)

    def close(self):
        for base in self._ipc:
            _check(lib().etg_ipc_close(ctypes.c_void_p(base)), "etg_ipc_close")
        self._ipc = []

    def run(self, alg: int, source: int = 0):
        return run_partitions([self.engine], self.group, alg, source, self.bounds, self.exchange)


class PushDistGraph:
    """This rank's SOURCE partition of a graph (out-edges of its owned range),
    driven with the push exchange (``run_push``) over a torch.distributed group."""

    def __init__(self, off, col, w, n: int, rank: int, world: int, *, K: int = 32, flags: int = 0,
                 symmetric: bool = False, device="cuda", group=None, bounds=None, mode: str = "auto"):
        from . import csr_to_device
        self.n, self.rank, self.world, self.mode = n, rank, world, mode
        self.bounds = bounds if bounds is not None else partition_ranges(off, col, n, world, by="out")
        lo, hi = self.bounds[rank], self.bounds[rank + 1]
        loff, lcol, lw = partition_csr_src(off, col, w, n, lo, hi)
        o, c, ww, fl = csr_to_device(loff, lcol, lw, device=device)
        self.graph = Graph(o, c, ww, n=n, K=K, flags=flags | fl, symmetric=symmetric)
        self.engine = CudaEngine(self.graph)
        self.group = TorchDistGroup(group)
        self._ipc = []
        if mode == "p2p" and world > 1:
            self._ipc = open_peer_labels(self.engine, self.bounds, rank, world, group)

    def close(self):
        for base in self._ipc:
            _check(lib().etg_ipc_close(ctypes.c_void_p(base)), "etg_ipc_close")
        self._ipc = []

    def run(self, alg: int, source: int = 0):
        labels, st, _ = run_push([self.engine], self.group, alg, source, self.bounds, [self.rank], self.mode)
        return labels, st
