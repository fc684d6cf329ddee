"""etg -- B200-native EtaGraph frontier expansion (BFS / SSSP / CC / SSWP).

Thin Python binding over the C ABI in ``include/etg.h`` (``libetg.so``, built
in-tree for sm_100a by ``_build.py``).  This module only marshals arguments:
every step of the traversal runs in the library's CUDA kernels.  There is no
CPU fallback -- if the library cannot be loaded or no CUDA device is present,
the calls raise.

Tensors are torch tensors on the CUDA device (PyTorch is used for device
memory and streams only).  Unsigned 32-bit arrays are carried in ``torch.int32``
tensors with the same bits (``labels.view(torch.int32)``); use
:func:`to_u32_numpy` to read them as ``uint32``.
"""
from __future__ import annotations

import ctypes
import os
from typing import Optional

import numpy as np
import torch

__all__ = [
    "EtgError", "Stats", "Graph", "load_csr", "csr_to_device", "to_u32_numpy",
    "run_host", "run_host_batch", "host_scratch_bytes", "kernel_launches", "lib", "Comm",
    "SYMMETRIC", "NO_UDC", "NO_SMP", "OFFSETS_U64", "VALIDATE", "HOST_LOOP", "PROFILE", "SMP_SHARED",
    "HOST_EDGES", "PUSH",
    "INF", "CAP", "BFS", "SSSP", "CC", "SSWP",
]

SYMMETRIC, NO_UDC, NO_SMP, OFFSETS_U64, VALIDATE, HOST_LOOP, PROFILE, SMP_SHARED, HOST_EDGES, PUSH = (
    1, 2, 4, 8, 16, 32, 64, 128, 256, 512)
INF, CAP = 0xFFFFFFFF, 0xFFFFFFFE
BFS, SSSP, CC, SSWP = 0, 1, 2, 3

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.environ.get("ETG_LIB_PATH") or os.path.join(_HERE, "libetg.so")
_lib = None


class EtgError(RuntimeError):
    pass


class Options(ctypes.Structure):
    _fields_ = [("degree_limit_k", ctypes.c_uint32), ("flags", ctypes.c_uint32),
                ("sssp_delta", ctypes.c_uint32)]


class Stats(ctypes.Structure):
    _fields_ = [
        ("iterations", ctypes.c_uint32), ("expand_launches", ctypes.c_uint32),
        ("activations", ctypes.c_uint64), ("frontier_total", ctypes.c_uint64),
        ("shadows", ctypes.c_uint64), ("edges_processed", ctypes.c_uint64),
        ("vertices_reached", ctypes.c_uint64), ("edges_reached", ctypes.c_uint64),
        ("ms", ctypes.c_float), ("scan_ms", ctypes.c_float), ("expand_ms", ctypes.c_float),
        ("reserved", ctypes.c_float),
    ]

    def asdict(self):
        return {k: getattr(self, k) for k, _ in self._fields_ if k != "reserved"}


def lib():
    """Load libetg.so (built by ``__graft_entry__.build()``); raise if absent."""
    global _lib
    if _lib is None:
        if not os.path.exists(_LIB_PATH):
            raise EtgError(f"{_LIB_PATH} is missing: run __graft_entry__.build() (no CPU fallback)")
        L = ctypes.CDLL(_LIB_PATH)
        p, u32, u64, sz = ctypes.c_void_p, ctypes.c_uint32, ctypes.c_uint64, ctypes.c_size_t
        st = ctypes.c_int
        sig = {
            "etg_workspace_bytes": (sz, [u64, u64, p]),
            "etg_load_csr": (st, [ctypes.POINTER(p), u64, u64, p, p, p, p, sz, p, p, p, u32, u32]),
            "etg_comm_unique_id": (st, [p]),
            "etg_comm_init": (st, [ctypes.POINTER(p), ctypes.c_int, ctypes.c_int, p, ctypes.c_int]),
            "etg_comm_barrier": (st, [p]),
            "etg_comm_free": (None, [p]),
            "etg_bfs": (st, [p, u32, p, p]),
            "etg_sssp": (st, [p, u32, p, p]),
            "etg_cc": (st, [p, p, p]),
            "etg_sswp": (st, [p, u32, p, p]),
            "etg_reach_stats": (st, [p, p, u32, p]),
            "etg_udc_slices": (st, [p, p, u32, p, p, p, u64, ctypes.POINTER(u64)]),
            "etg_free": (None, [p]),
            "etg_host_scratch_bytes": (sz, [u64, u64, ctypes.c_int, p]),
            "etg_run_host": (st, [ctypes.c_int, u64, u64, p, p, p, u32, p, p, sz, p, p, p]),
            "etg_run_host_batch": (st, [u64, u64, p, p, p, u32, p, p, p, p, sz, p, p, p]),
            "etg_status_str": (ctypes.c_char_p, [st]),
            "etg_last_error": (ctypes.c_char_p, []),
            "etg_kernel_launches": (u64, []),
            "etg_step_begin": (st, [p, ctypes.c_int, u32, p, ctypes.POINTER(u32)]),
            "etg_step_expand": (st, [p]),
            "etg_debug_counters": (st, [p, ctypes.POINTER(ctypes.c_uint64)]),
            "etg_step_scan": (st, [p, ctypes.POINTER(u32)]),
            "etg_step_end": (st, [p, p]),
            "etg_bitmap_layout": (st, [p, ctypes.POINTER(sz), ctypes.POINTER(u32)]),
            "etg_sssp_delta": (st, [p, ctypes.POINTER(u32)]),
            "etg_debug_expand_replay": (st, [p, ctypes.c_int, u32, u32, u32, ctypes.c_int, p, p,
                                             ctypes.POINTER(ctypes.c_float), ctypes.POINTER(u64),
                                             ctypes.POINTER(u32)]),
        }
        for name, (res, args) in sig.items():
            f = getattr(L, name)
            f.restype = res
            f.argtypes = args
        _lib = L
    return _lib


SSSP_DELTA_AUTO = 0xFFFFFFFF


def _delta(d) -> int:
    """sssp_delta: an int (0 = the paper's schedule) or "auto" (6 x mean edge
    weight / mean out-degree, at least 1: 12 / 13 / 6 on C2 / C3 / C4)."""
    return SSSP_DELTA_AUTO if d == "auto" else int(d)


def _check(rc: int, what: str):
    if rc != 0:
        L = lib()
        raise EtgError(f"{what}: {L.etg_status_str(rc).decode()} ({L.etg_last_error().decode()})")


def _ptr(t: Optional[torch.Tensor]):
    return None if t is None else ctypes.c_void_p(t.data_ptr())


def _stream_ptr(stream) -> ctypes.c_void_p:
    s = stream if stream is not None else torch.cuda.current_stream()
    return ctypes.c_void_p(s.cuda_stream)


def kernel_launches() -> int:
    """CUDA kernels launched by libetg.so in this process so far."""
    return int(lib().etg_kernel_launches())


def to_u32_numpy(t: torch.Tensor) -> np.ndarray:
    return t.detach().cpu().numpy().view(np.uint32)


def _as_u32_bits(x: torch.Tensor) -> torch.Tensor:
    """int64 values in [0, 2^32) -> int32 tensor holding the same 32 bits."""
    x = x.to(torch.int64)
    return torch.where(x >= (1 << 31), x - (1 << 32), x).to(torch.int32).contiguous()


def csr_to_device(off: torch.Tensor, col: torch.Tensor, w: Optional[torch.Tensor] = None,
                  device="cuda"):
    """(off, col, w) of any integer dtype -> device tensors in the library layout.

    Returns (off, col, w, flags): off is uint32-in-int32 when m < 2^32, else int64
    (ETG_OFFSETS_U64); col and w are uint32-in-int32.
    """
    m = int(col.shape[0])
    flags = 0
    off = off.to(device)
    if m < (1 << 32):
        off_d = _as_u32_bits(off)
    else:
        off_d = off.to(torch.int64).contiguous()
        flags |= OFFSETS_U64
    col_d = _as_u32_bits(col.to(device))
    w_d = None if w is None else _as_u32_bits(w.to(device))
    return off_d, col_d, w_d, flags


class Comm:
    """A communicator over the ranks of one node (etg_comm_init).  Rank 0 makes
    the id with :meth:`unique_id`; the caller hands it to the other ranks
    (e.g. torch.distributed.broadcast_object_list -- bootstrap only)."""

    def __init__(self, rank: int, world: int, uid: bytes, device: int = -1):
        if len(uid) != 128:
            raise EtgError("unique id must be 128 bytes")
        h = ctypes.c_void_p()
        _check(lib().etg_comm_init(ctypes.byref(h), rank, world, (ctypes.c_uint8 * 128)(*uid), device),
               "etg_comm_init")
        self._h = h
        self.rank, self.world, self.device = rank, world, device

    @staticmethod
    def unique_id() -> bytes:
        buf = (ctypes.c_uint8 * 128)()
        _check(lib().etg_comm_unique_id(buf), "etg_comm_unique_id")
        return bytes(buf)

    def barrier(self) -> None:
        _check(lib().etg_comm_barrier(self._h), "etg_comm_barrier")

    def close(self):
        if getattr(self, "_h", None):
            lib().etg_comm_free(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


class Graph:
    """A handle over a device CSR (etg_load_csr).  Keeps its tensors alive.

    With ``comm`` (a :class:`Comm`): this rank's partition of a graph of ``n``
    vertices owning [v_lo, v_hi) (see include/etg.h); construction is
    collective, every traversal is collective and returns the owned slice."""

    def __init__(self, off: torch.Tensor, col: torch.Tensor, w: Optional[torch.Tensor] = None, *,
                 n: Optional[int] = None, K: int = 32, flags: int = 0, symmetric: bool = False,
                 validate: bool = False, stream=None, sssp_delta: int = 0, comm: Optional[Comm] = None,
                 v_lo: int = 0, v_hi: Optional[int] = None):
        if not torch.cuda.is_available():
            raise EtgError("no CUDA device: etg has no CPU fallback")
        if off.dtype == torch.int64:
            flags |= OFFSETS_U64
        elif off.dtype != torch.int32:
            raise EtgError("row offsets must be int32 (u32 bits) or int64")
        if col.dtype != torch.int32 or (w is not None and w.dtype != torch.int32):
            raise EtgError("col and w must be int32 tensors holding uint32 bits")
        for t in (off, col, w):
            if t is None:
                continue
            edge_array = t is not off
            host_ok = edge_array and (flags & HOST_EDGES) and t.is_pinned()
            if not t.is_contiguous() or not (t.is_cuda or host_ok):
                raise EtgError("CSR tensors must be contiguous CUDA tensors "
                               "(col/w may be pinned host tensors with HOST_EDGES)")
        if symmetric:
            flags |= SYMMETRIC
        if validate:
            flags |= VALIDATE
        self.n = int(off.shape[0] - 1) if n is None else n
        self.m = int(col.shape[0])
        self.K = K
        self.flags = flags
        self.device = off.device
        if not off.is_cuda:
            raise EtgError("row offsets must live on the device")
        self._keep = (off, col, w, comm)
        self._stream = stream
        self.comm = comm
        self.v_lo = v_lo if comm is not None else 0
        self.v_hi = (self.n if v_hi is None else v_hi) if comm is not None else self.n
        self._opt = Options(K, flags, _delta(sssp_delta))
        L = lib()
        nbytes = L.etg_workspace_bytes(self.n, self.m, ctypes.byref(self._opt))
        self.workspace = torch.empty(max(nbytes, 256), dtype=torch.uint8, device=self.device)
        h = ctypes.c_void_p()
        rc = L.etg_load_csr(ctypes.byref(h), self.n, self.m, _ptr(off), _ptr(col), _ptr(w),
                            _ptr(self.workspace), nbytes, _stream_ptr(stream),
                            ctypes.byref(self._opt), None if comm is None else comm._h,
                            self.v_lo, self.v_hi)
        _check(rc, "etg_load_csr")
        self._h = h

    # -- traversals --------------------------------------------------------- #
    def _out(self, out):
        k = self.v_hi - self.v_lo            # n, or the owned slice of a partition
        if out is None:
            out = torch.empty(max(k, 1), dtype=torch.int32, device=self.device)
        if out.dtype != torch.int32 or out.numel() < k or not out.is_contiguous():
            raise EtgError(f"out must be a contiguous int32 tensor of {k} entries")
        return out

    def bfs(self, source: int, out: Optional[torch.Tensor] = None):
        out = self._out(out)
        st = Stats()
        _check(lib().etg_bfs(self._h, source, _ptr(out), ctypes.byref(st)), "etg_bfs")
        return out, st

    def sssp(self, source: int, out: Optional[torch.Tensor] = None):
        out = self._out(out)
        st = Stats()
        _check(lib().etg_sssp(self._h, source, _ptr(out), ctypes.byref(st)), "etg_sssp")
        return out, st

    def cc(self, out: Optional[torch.Tensor] = None):
        out = self._out(out)
        st = Stats()
        _check(lib().etg_cc(self._h, _ptr(out), ctypes.byref(st)), "etg_cc")
        return out, st

    def sswp(self, source: int, out: Optional[torch.Tensor] = None):
        out = self._out(out)
        st = Stats()
        _check(lib().etg_sswp(self._h, source, _ptr(out), ctypes.byref(st)), "etg_sswp")
        return out, st

    def run(self, alg: int, source: int = 0, out=None):
        if alg == BFS:
            return self.bfs(source, out)
        if alg == SSSP:
            return self.sssp(source, out)
        if alg == CC:
            return self.cc(out)
        return self.sswp(source, out)

    def sssp_delta(self) -> int:
        """The SSSP wave width Delta of this handle (auto resolved on first use)."""
        d = ctypes.c_uint32()
        _check(lib().etg_sssp_delta(self._h, ctypes.byref(d)), "etg_sssp_delta")
        return int(d.value)

    def reach_stats(self, labels: torch.Tensor, unreached: int = INF) -> Stats:
        st = Stats()
        _check(lib().etg_reach_stats(self._h, _ptr(labels), unreached, ctypes.byref(st)),
               "etg_reach_stats")
        return st

    def udc_slices(self, active: torch.Tensor):
        """Step A2 through the library's device mapping: (ids, start, end) tensors."""
        active = active.to(torch.int32).contiguous()
        L = lib()
        cap = ctypes.c_uint64(0)
        n_act = int(active.numel())
        ids = torch.empty(1, dtype=torch.int32, device=self.device)
        st = torch.empty(1, dtype=torch.int64, device=self.device)
        en = torch.empty(1, dtype=torch.int64, device=self.device)
        rc = L.etg_udc_slices(self._h, _ptr(active), n_act, _ptr(ids), _ptr(st), _ptr(en), 0,
                              ctypes.byref(cap))
        if rc not in (0, -2):
            _check(rc, "etg_udc_slices")
        cnt = int(cap.value)
        ids = torch.empty(max(cnt, 1), dtype=torch.int32, device=self.device)
        st = torch.empty(max(cnt, 1), dtype=torch.int64, device=self.device)
        en = torch.empty(max(cnt, 1), dtype=torch.int64, device=self.device)
        out = ctypes.c_uint64(0)
        _check(L.etg_udc_slices(self._h, _ptr(active), n_act, _ptr(ids), _ptr(st), _ptr(en),
                                cnt, ctypes.byref(out)), "etg_udc_slices")
        return ids[:cnt], st[:cnt], en[:cnt]

    def debug_expand_replay(self, alg: int, source: int, depth: int, tune: int = 0, reps: int = 5):
        """Time the expand kernel on the snapshot of iteration `depth` (tuning aid)."""
        lab = torch.empty(self.n, dtype=torch.int32, device=self.device)
        saved = torch.empty(self.n, dtype=torch.int32, device=self.device)
        ms, edges, nact = ctypes.c_float(), ctypes.c_uint64(), ctypes.c_uint32()
        _check(lib().etg_debug_expand_replay(self._h, alg, source, depth, tune, reps, _ptr(lab),
                                             _ptr(saved), ctypes.byref(ms), ctypes.byref(edges),
                                             ctypes.byref(nact)), "etg_debug_expand_replay")
        return ms.value, int(edges.value), int(nact.value)

    def close(self):
        if getattr(self, "_h", None):
            lib().etg_free(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def load_csr(off, col, w=None, **kw) -> Graph:
    return Graph(off, col, w, **kw)


def host_scratch_bytes(n: int, m: int, has_weights: bool, K: int = 32, flags: int = 0) -> int:
    opt = Options(K, flags, 0)
    return int(lib().etg_host_scratch_bytes(n, m, int(has_weights), ctypes.byref(opt)))


def run_host(alg: int, off: torch.Tensor, col: torch.Tensor, w: Optional[torch.Tensor],
             source: int, labels_out: torch.Tensor, scratch: torch.Tensor, *, K: int = 32,
             flags: int = 0, stream=None, sssp_delta: int = 0, symmetric: bool = False) -> Stats:
    """End-to-end call on HOST tensors (pinned recommended): H2D, traverse, D2H.
    CC needs ``symmetric=True`` (the caller asserts the CSR is symmetric, as
    with :class:`Graph`); without it the library returns ETG_ENOTSYM."""
    for t in (off, col, w, labels_out):
        if t is not None and t.is_cuda:
            raise EtgError("run_host takes host tensors")
    if off.dtype == torch.int64:
        flags |= OFFSETS_U64
    if symmetric:
        flags |= SYMMETRIC
    n = int(off.shape[0] - 1)
    m = int(col.shape[0])
    opt = Options(K, flags, _delta(sssp_delta))
    st = Stats()
    rc = lib().etg_run_host(alg, n, m, _ptr(off), _ptr(col), _ptr(w), source, _ptr(labels_out),
                            _ptr(scratch), scratch.numel() * scratch.element_size(),
                            _stream_ptr(stream), ctypes.byref(opt), ctypes.byref(st))
    _check(rc, "etg_run_host")
    return st


def run_host_batch(queries, off: torch.Tensor, col: torch.Tensor, w: Optional[torch.Tensor],
                   labels_out: torch.Tensor, scratch: torch.Tensor, *, K: int = 32, flags: int = 0,
                   stream=None, sssp_delta: int = 0, symmetric: bool = False):
    """Several traversals of one HOST graph, the CSR copied once:
    ``queries`` = [(alg, source), ...]; ``labels_out`` a host int32 tensor of
    len(queries) x n.  Returns the list of Stats."""
    for t in (off, col, w, labels_out):
        if t is not None and t.is_cuda:
            raise EtgError("run_host_batch takes host tensors")
    if off.dtype == torch.int64:
        flags |= OFFSETS_U64
    if symmetric:
        flags |= SYMMETRIC
    n = int(off.shape[0] - 1)
    m = int(col.shape[0])
    q = len(queries)
    if labels_out.numel() < q * n or labels_out.dtype != torch.int32 or not labels_out.is_contiguous():
        raise EtgError("labels_out must be a contiguous int32 host tensor of len(queries) x n")
    algs = (ctypes.c_int * q)(*[a for a, _ in queries])
    srcs = (ctypes.c_uint32 * q)(*[s for _, s in queries])
    opt = Options(K, flags, _delta(sssp_delta))
    sts = (Stats * q)()
    rc = lib().etg_run_host_batch(n, m, _ptr(off), _ptr(col), _ptr(w), q, algs, srcs, _ptr(labels_out),
                                  _ptr(scratch), scratch.numel() * scratch.element_size(),
                                  _stream_ptr(stream), ctypes.byref(opt), sts)
    _check(rc, "etg_run_host_batch")
    return list(sts)
