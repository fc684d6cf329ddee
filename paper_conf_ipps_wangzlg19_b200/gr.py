"""Galois binary CSR (`.gr`) reader/writer -- the on-disk format EtaGraph loads
("We use Galois CSR binary format to store graph data for
loading from disk").

Layout (little-endian), version 1 (32-bit node ids) or 2 (64-bit node ids):

    uint64 version, uint64 sizeof_edge_data, uint64 num_nodes, uint64 num_edges
    uint64 out_idx[num_nodes]        -- END offset of each node's edge list
    uint{32|64} outs[num_edges]      -- destination ids
    [uint32 pad]                     -- v1 only, when num_edges is odd (8-byte alignment)
    edge_data[num_edges]             -- sizeof_edge_data bytes each (here 0 or 4: uint32 weights)

Host-side I/O only (numpy memory maps); the arrays go to the device through
``csr_to_device`` like any other CSR.
"""
from __future__ import annotations

import os
from typing import Optional, Tuple

import numpy as np


def read_gr(path: str) -> Tuple[np.ndarray, np.ndarray, Optional[np.ndarray]]:
    """Return (off int64[n+1], col uint32[m], w uint32[m] or None)."""
    hdr = np.fromfile(path, dtype="<u8", count=4)
    if hdr.shape[0] != 4:
        raise ValueError(f"{path}: truncated header")
    version, esize, n, m = (int(x) for x in hdr)
    if version not in (1, 2):
        raise ValueError(f"{path}: unsupported .gr version {version}")
    if esize not in (0, 4):
        raise ValueError(f"{path}: edge data of {esize} bytes (only none or uint32 supported)")
    mm = np.memmap(path, dtype=np.uint8, mode="r")
    pos = 32
    ends = np.frombuffer(mm, dtype="<u8", count=n, offset=pos)
    pos += 8 * n
    idt = "<u4" if version == 1 else "<u8"
    isz = 4 if version == 1 else 8
    outs = np.frombuffer(mm, dtype=idt, count=m, offset=pos)
    pos += isz * m
    if version == 1 and m % 2:
        pos += 4
    w = None
    if esize:
        w = np.array(np.frombuffer(mm, dtype="<u4", count=m, offset=pos), dtype=np.uint32)
        pos += 4 * m
    if pos != os.path.getsize(path):
        raise ValueError(f"{path}: size {os.path.getsize(path)} != expected {pos}")
    off = np.zeros(n + 1, dtype=np.int64)
    off[1:] = ends.astype(np.int64)
    if n and (np.any(np.diff(off) < 0) or off[-1] != m):
        raise ValueError(f"{path}: malformed offsets")
    if m and int(outs.max()) >= n:
        raise ValueError(f"{path}: destination id out of range")
    return off, np.array(outs, dtype=np.uint32), w


def write_gr(path: str, off, col, w=None, version: int = 1) -> None:
    """Write a CSR as a Galois .gr file (version 1: 32-bit ids, 2: 64-bit ids)."""
    off = np.asarray(off, dtype=np.int64)
    col = np.asarray(col)
    n, m = off.shape[0] - 1, col.shape[0]
    with open(path, "wb") as f:
        np.array([version, 4 if w is not None else 0, n, m], dtype="<u8").tofile(f)
        off[1:].astype("<u8").tofile(f)
        col.astype("<u4" if version == 1 else "<u8").tofile(f)
        if version == 1 and m % 2:
            np.zeros(1, dtype="<u4").tofile(f)
        if w is not None:
            np.asarray(w).astype("<u4").tofile(f)
