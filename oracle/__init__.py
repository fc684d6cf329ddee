"""CPU oracle for the EtaGraph hot path -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` legs may import this package.  The product path
(``paper_conf_ipps_wangzlg19_b200``) never imports it and shares no code with it.

The arithmetic lives in ``oracle.c`` (plain C, single thread); this module only
compiles it with gcc (on first use, or from ``__graft_entry__.build()``) and
marshals numpy arrays through ctypes.  See ``oracle.c`` for the passage of
PAPER.md each function follows.  Every function is pinned by
``tests/test_oracle_*.py`` (closed forms, brute force, scipy/networkx,
certificates, the golden fixtures under ``tests/golden/``).
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import threading

import numpy as np

INF = 0xFFFFFFFF
CAP = 0xFFFFFFFE

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB = os.path.join(_HERE, "_oracle.so")
_lock = threading.Lock()
_lib = None


def build(force: bool = False) -> str:
    """Compile oracle.c into _oracle.so with gcc (-O3, single-threaded; no
    -march=native: the library built here also runs on the GPU box's host CPU)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O3", "-std=c99", "-shared", "-fPIC", _SRC, "-o", tmp])
        os.replace(tmp, _LIB)
    return _LIB


def _load():
    global _lib
    with _lock:
        if _lib is None:
            build()
            lib = ctypes.CDLL(_LIB)
            u64, p = ctypes.c_uint64, ctypes.c_void_p
            for name, args in (
                ("oracle_bfs", [u64, p, p, ctypes.c_uint32, p]),
                ("oracle_sssp", [u64, p, p, p, ctypes.c_uint32, p]),
                ("oracle_sswp", [u64, p, p, p, ctypes.c_uint32, p]),
                ("oracle_cc", [u64, p, p, p]),
            ):
                f = getattr(lib, name)
                f.argtypes = args
                f.restype = ctypes.c_int
            f = lib.oracle_udc_slices
            f.argtypes = [u64, p, p, u64, u64, p, p, p, u64]
            f.restype = ctypes.c_int64
            _lib = lib
    return _lib


def _ptr(a: np.ndarray):
    return a.ctypes.data_as(ctypes.c_void_p)


def _csr(off, col, w=None):
    off = np.ascontiguousarray(off, dtype=np.uint64)
    col = np.ascontiguousarray(col, dtype=np.uint32)
    n = off.shape[0] - 1
    if n < 0 or int(off[-1]) != col.shape[0]:
        raise ValueError("bad CSR")
    if w is not None:
        w = np.ascontiguousarray(w, dtype=np.uint32)
        if w.shape[0] != col.shape[0]:
            raise ValueError("weights length != m")
    return n, off, col, w


def bfs(off, col, source: int) -> np.ndarray:
    """Hop depth from ``source``; INF for unreachable (oracle.c: oracle_bfs)."""
    n, off, col, _ = _csr(off, col)
    out = np.empty(n, dtype=np.uint32)
    rc = _load().oracle_bfs(n, _ptr(off), _ptr(col), source, _ptr(out))
    if rc:
        raise ValueError(f"oracle_bfs rc={rc}")
    return out


def sssp(off, col, w, source: int) -> np.ndarray:
    """Saturating shortest distance (CAP), INF unreachable (oracle.c: oracle_sssp)."""
    n, off, col, w = _csr(off, col, w)
    out = np.empty(n, dtype=np.uint32)
    rc = _load().oracle_sssp(n, _ptr(off), _ptr(col), _ptr(w), source, _ptr(out))
    if rc:
        raise ValueError(f"oracle_sssp rc={rc}")
    return out


def sswp(off, col, w, source: int) -> np.ndarray:
    """Widest-path width (INF at source, 0 unreachable) (oracle.c: oracle_sswp)."""
    n, off, col, w = _csr(off, col, w)
    out = np.empty(n, dtype=np.uint32)
    rc = _load().oracle_sswp(n, _ptr(off), _ptr(col), _ptr(w), source, _ptr(out))
    if rc:
        raise ValueError(f"oracle_sswp rc={rc}")
    return out


def cc(off, col) -> np.ndarray:
    """Minimum vertex id of each weakly connected component (oracle.c: oracle_cc)."""
    n, off, col, _ = _csr(off, col)
    out = np.empty(n, dtype=np.uint32)
    rc = _load().oracle_cc(n, _ptr(off), _ptr(col), _ptr(out))
    if rc:
        raise ValueError(f"oracle_cc rc={rc}")
    return out


def udc_slices(off, active, K: int):
    """Def. 3 shadow vertices of an active set: arrays (id, start, end) (oracle_udc_slices)."""
    off = np.ascontiguousarray(off, dtype=np.uint64)
    act = np.ascontiguousarray(active, dtype=np.uint32)
    n = off.shape[0] - 1
    lib = _load()
    cap = 1024
    while True:
        ids = np.empty(cap, dtype=np.uint32)
        st = np.empty(cap, dtype=np.uint64)
        en = np.empty(cap, dtype=np.uint64)
        rc = lib.oracle_udc_slices(n, _ptr(off), _ptr(act), act.shape[0], K,
                                   _ptr(ids), _ptr(st), _ptr(en), cap)
        if rc == -1:
            raise ValueError("bad udc input")
        if rc >= 0:
            return ids[:rc].copy(), st[:rc].copy(), en[:rc].copy()
        cap = -rc - 2
