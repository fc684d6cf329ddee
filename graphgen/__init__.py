"""Seeded synthetic graph generators shared by the oracle and the CUDA path.

This module holds INPUT GENERATION ONLY -- none of the method's arithmetic (no
traversal, no UDC, no relaxation).  Both sides of every parity test read the
same CSR produced here; neither side imports the other.

Design:

* randomness is counter-based: ``rand64(seed, i)`` is the SplitMix64 output for
  counter ``i`` (state = key + (i+1)*GAMMA, then the SplitMix64 finaliser), so
  any element can be regenerated independently, on any device;
* everything is integer arithmetic on int64 torch tensors (wrapping multiply,
  emulated logical shifts), so the CPU and CUDA builds of a graph are
  bit-identical (pinned by tests/test_graphgen.py against a numpy-uint64
  re-derivation and, on the GPU box, CPU-vs-CUDA);
* RMAT (PaRMAT parameters a/b/c = .45/.22/.22, d = .11) draws one
  32-bit uniform per recursion level and compares it with integer quadrant
  thresholds floor(p * 2^32);
* Chung-Lu power-law graphs (LiveJournal- and Twitter-shaped, PAPER.md
  Table II) sample endpoints through integer cumulative weights
  (float64 weights are computed on the host with numpy, then quantised);
* vertex ids are relabelled by a keyed 4-round Feistel permutation with
  cycle-walking, self-loops are dropped and duplicates removed (PAPER.md L119:
  "we consider graphs with no duplicate edges"); the CSR is sorted by (src, dst);
* SSSP weights are ``1 + rand64(wseed, (u << 32) | v) mod wmax`` -- a function
  of the final endpoint ids (reading R-8), uint32, one array beside ``col``.
"""
from __future__ import annotations

import dataclasses
import hashlib
import math
from typing import Optional

import numpy as np
import torch

M64 = (1 << 64) - 1
GAMMA = 0x9E3779B97F4A7C15
MIX1 = 0xBF58476D1CE4E5B9
MIX2 = 0x94D049BB133111EB


def _s64(x: int) -> int:
    """Unsigned 64-bit constant -> the int64 with the same bits."""
    x &= M64
    return x - (1 << 64) if x >= (1 << 63) else x


_GAMMA_S, _MIX1_S, _MIX2_S = _s64(GAMMA), _s64(MIX1), _s64(MIX2)


def _srl(x: torch.Tensor, s: int) -> torch.Tensor:
    """Logical right shift of int64 bits."""
    return (x >> s) & ((1 << (64 - s)) - 1)


def mix64(z: torch.Tensor) -> torch.Tensor:
    """SplitMix64 finaliser on int64 tensors (wrapping arithmetic)."""
    z = (z ^ _srl(z, 30)) * _MIX1_S
    z = (z ^ _srl(z, 27)) * _MIX2_S
    return z ^ _srl(z, 31)


def seed_key(seed: int, stream: int = 0) -> int:
    """Derive a 64-bit key for (seed, stream); pure-python, exact."""
    z = (seed * 0xD1B54A32D192ED03 + stream * GAMMA + 0x632BE59BD9B4E019) & M64
    z = ((z ^ (z >> 30)) * MIX1) & M64
    z = ((z ^ (z >> 27)) * MIX2) & M64
    return _s64(z ^ (z >> 31))


def rand64(key: int, ctr: torch.Tensor) -> torch.Tensor:
    """Counter-based 64-bit random words: SplitMix64 output number ``ctr``."""
    return mix64(key + (ctr + 1) * _GAMMA_S)


# numpy-uint64 re-derivation used only by tests to pin the torch arithmetic.
def rand64_numpy(key: int, ctr: np.ndarray) -> np.ndarray:
    with np.errstate(over="ignore"):
        z = np.uint64(key & M64) + (ctr.astype(np.uint64) + np.uint64(1)) * np.uint64(GAMMA)
        z = (z ^ (z >> np.uint64(30))) * np.uint64(MIX1)
        z = (z ^ (z >> np.uint64(27))) * np.uint64(MIX2)
        return z ^ (z >> np.uint64(31))


# --------------------------------------------------------------------------- #
# Feistel permutation of [0, n) (cycle-walking), keyed
# --------------------------------------------------------------------------- #
def feistel_permute(x: torch.Tensor, n: int, key: int, rounds: int = 4) -> torch.Tensor:
    """Keyed bijection of [0, n) applied elementwise to ``x`` (int64)."""
    if n <= 1:
        return x.clone()
    bits = max(2, (n - 1).bit_length())
    bits += bits & 1
    half = bits // 2
    mask = (1 << half) - 1
    rkeys = [seed_key(key, 1000 + r) for r in range(rounds)]

    def once(y):
        lo, hi = y & mask, y >> half
        for rk in rkeys:
            f = rand64(rk, lo) & mask
            lo, hi = hi ^ f, lo
        return (hi << half) | lo

    y = once(x)
    bad = y >= n
    while bool(bad.any()):
        y = torch.where(bad, once(y), y)
        bad = y >= n
    return y


# --------------------------------------------------------------------------- #
# CSR container
# --------------------------------------------------------------------------- #
@dataclasses.dataclass
class Graph:
    """A CSR graph: ``off`` int64[n+1], ``col`` int64[m], ``w`` int64[m] or None."""
    name: str
    n: int
    off: torch.Tensor
    col: torch.Tensor
    w: Optional[torch.Tensor] = None
    symmetric: bool = False

    @property
    def m(self) -> int:
        return int(self.col.shape[0])

    def to(self, device) -> "Graph":
        return Graph(self.name, self.n, self.off.to(device), self.col.to(device),
                     None if self.w is None else self.w.to(device), self.symmetric)

    def numpy(self):
        """(off uint64, col uint32, w uint32|None) host arrays for the oracle."""
        off = self.off.cpu().numpy().astype(np.uint64)
        col = self.col.cpu().numpy().astype(np.uint32)
        w = None if self.w is None else self.w.cpu().numpy().astype(np.uint32)
        return off, col, w

    def sha256(self) -> str:
        h = hashlib.sha256()
        off, col, w = self.numpy()
        h.update(off.tobytes())
        h.update(col.tobytes())
        if w is not None:
            h.update(w.tobytes())
        return h.hexdigest()

    def degrees(self) -> torch.Tensor:
        return self.off[1:] - self.off[:-1]


def csr_from_keys(name: str, n: int, keys: torch.Tensor) -> Graph:
    """Sorted unique keys src*n+dst -> CSR (drops nothing; caller dedups)."""
    src = torch.div(keys, n, rounding_mode="floor")
    dst = keys - src * n
    cnt = torch.bincount(src, minlength=n)
    off = torch.zeros(n + 1, dtype=torch.int64, device=keys.device)
    off[1:] = torch.cumsum(cnt, 0)
    return Graph(name, n, off, dst)


_BUCKET_TUPLES = 1 << 27      # tuples per dedup bucket (tests lower it)


class KeyBuckets:
    """Accumulates (src, dst) tuples chunk by chunk, routed into source-range
    buckets, so large graphs are deduplicated bucket by bucket (never one sort
    of all tuples); concatenating the buckets in order keeps the CSR sorted."""

    def __init__(self, n: int, total: int):
        self.n = n
        want = max(1, min(n, -(-total // _BUCKET_TUPLES)))      # buckets needed
        self.shift = max(0, (max(n - 1, 1) // want).bit_length()) if want > 1 else 64
        self.nb = 1 if want == 1 else ((n - 1) >> self.shift) + 1
        self.parts = [[] for _ in range(self.nb)]

    def add(self, src: torch.Tensor, dst: torch.Tensor) -> None:
        keys = dedup_keys(src, dst, self.n)
        if self.nb == 1:
            self.parts[0].append(keys)
            return
        b = torch.div(keys, self.n, rounding_mode="floor") >> self.shift
        bounds = torch.searchsorted(b, torch.arange(self.nb + 1, device=b.device))
        for i in range(self.nb):
            lo, hi = int(bounds[i]), int(bounds[i + 1])
            if hi > lo:
                self.parts[i].append(keys[lo:hi])

    def csr(self, name: str, device) -> "Graph":
        cnt = torch.zeros(self.n, dtype=torch.int64, device=device)
        cols = []
        for i in range(self.nb):
            if not self.parts[i]:
                continue
            k = torch.unique(torch.cat(self.parts[i]), sorted=True)
            self.parts[i] = None
            src = torch.div(k, self.n, rounding_mode="floor")
            cnt += torch.bincount(src, minlength=self.n)
            cols.append(k - src * self.n)
            del k, src
        off = torch.zeros(self.n + 1, dtype=torch.int64, device=device)
        off[1:] = torch.cumsum(cnt, 0)
        col = torch.cat(cols) if cols else torch.zeros(0, dtype=torch.int64, device=device)
        return Graph(name, self.n, off, col)


def dedup_keys(src: torch.Tensor, dst: torch.Tensor, n: int) -> torch.Tensor:
    keep = src != dst                                     # drop self-loops
    keys = src[keep] * n + dst[keep]
    return torch.unique(keys, sorted=True)


def edge_list(g: Graph):
    src = torch.repeat_interleave(torch.arange(g.n, device=g.off.device), g.degrees())
    return src, g.col


def from_edges(name: str, n: int, edges, *, weights=None, dedup: bool = False,
               device="cpu") -> Graph:
    """Tiny hand-built graphs: a list of (u, v) -> CSR sorted by (u, v), stable.

    Keeps duplicates and self-loops unless ``dedup`` (the fixtures need both).
    """
    e = np.asarray(edges, dtype=np.int64).reshape(-1, 2)
    order = np.lexsort((e[:, 1], e[:, 0])) if len(e) else np.zeros(0, dtype=np.int64)
    e = e[order]
    w = None
    if weights is not None:
        w = np.asarray(weights, dtype=np.int64)[order]
    if dedup and len(e):
        keep = np.ones(len(e), dtype=bool)
        keep[1:] = np.any(e[1:] != e[:-1], axis=1)
        keep &= e[:, 0] != e[:, 1]
        e = e[keep]
        if w is not None:
            w = w[keep]
    cnt = np.bincount(e[:, 0], minlength=n) if len(e) else np.zeros(n, dtype=np.int64)
    off = np.zeros(n + 1, dtype=np.int64)
    off[1:] = np.cumsum(cnt)
    t = lambda a: torch.from_numpy(np.ascontiguousarray(a)).to(device)
    return Graph(name, n, t(off), t(e[:, 1].copy()), None if w is None else t(w))


def add_weights(g: Graph, seed: int, wmax: int = 64) -> Graph:
    """Reading R-8: w(u,v) = 1 + (rand64(wkey, (u<<32)|v) >> 1) mod wmax."""
    src, dst = edge_list(g)
    h = _srl(rand64(seed_key(seed, 7), (src << 32) | dst), 1)
    w = 1 + torch.remainder(h, wmax)
    return Graph(g.name, g.n, g.off, g.col, w, g.symmetric)


def symmetrize(g: Graph) -> Graph:
    """Union of E and its reverse, deduplicated, self-loops dropped (CC input, R-10)."""
    src, dst = edge_list(g)
    keys = dedup_keys(torch.cat([src, dst]), torch.cat([dst, src]), g.n)
    out = csr_from_keys(g.name + "-sym", g.n, keys)
    out.symmetric = True
    return out


# --------------------------------------------------------------------------- #
# RMAT (PaRMAT parameters)
# --------------------------------------------------------------------------- #
def rmat(scale: int, edge_factor: int = 16, a: float = 0.45, b: float = 0.22,
         c: float = 0.22, seed: int = 16, device="cpu", chunk: int = 1 << 24,
         name: Optional[str] = None, permute: bool = True) -> Graph:
    n = 1 << scale
    ntup = edge_factor << scale
    tA = int(math.floor(a * 2**32))
    tAB = int(math.floor((a + b) * 2**32))
    tABC = int(math.floor((a + b + c) * 2**32))
    key = seed_key(seed, 1)
    pkey = seed_key(seed, 2)
    acc = KeyBuckets(n, ntup)
    words = (scale + 1) // 2
    for lo in range(0, ntup, chunk):
        e = torch.arange(lo, min(ntup, lo + chunk), dtype=torch.int64, device=device)
        src = torch.zeros_like(e)
        dst = torch.zeros_like(e)
        for wd in range(words):
            r = rand64(key, e * 16 + wd)
            for half in range(2):
                lvl = 2 * wd + half
                if lvl >= scale:
                    break
                u = _srl(r, 32 * half) & 0xFFFFFFFF if half else r & 0xFFFFFFFF
                sbit = (u >= tAB).to(torch.int64)
                dbit = (((u >= tA) & (u < tAB)) | (u >= tABC)).to(torch.int64)
                bit = scale - 1 - lvl
                src |= sbit << bit
                dst |= dbit << bit
        if permute:
            src = feistel_permute(src, n, pkey)
            dst = feistel_permute(dst, n, pkey)
        acc.add(src, dst)
        del e, src, dst
    return acc.csr(name or f"rmat{scale}", device)


# --------------------------------------------------------------------------- #
# Chung-Lu power law (LiveJournal- / Twitter-shaped)
# --------------------------------------------------------------------------- #
def _powerlaw_weights(n: int, alpha: float, dmax: float, total: float) -> np.ndarray:
    """d_i = c (i + i0)^-beta, beta = 1/(alpha-1), with d_0 = dmax and sum = total."""
    beta = 1.0 / (alpha - 1.0)
    i = np.arange(n, dtype=np.float64)

    def ssum(i0):
        return float(np.sum((i + i0) ** -beta)) * dmax * i0 ** beta

    lo, hi = 1e-3, 1e9
    for _ in range(200):                     # sum is increasing in i0: bisection
        mid = math.sqrt(lo * hi)
        if ssum(mid) < total:
            lo = mid
        else:
            hi = mid
    i0 = math.sqrt(lo * hi)
    return dmax * (i0 ** beta) * (i + i0) ** -beta


def chung_lu(n: int, m_target: int, alpha_out: float, dmax_out: float,
             alpha_in: float, dmax_in: float, oversample: float, seed: int,
             device="cpu", chunk: int = 1 << 24, name: str = "chunglu") -> Graph:
    ntup = int(round(m_target * oversample))
    cum = []
    for alpha, dmax in ((alpha_out, dmax_out), (alpha_in, dmax_in)):
        wts = _powerlaw_weights(n, alpha, dmax, float(m_target))
        q = np.maximum(np.round(wts * 1024.0), 1).astype(np.int64)   # integer weights
        cum.append(torch.from_numpy(np.cumsum(q)).to(device))
    key_s, key_d = seed_key(seed, 3), seed_key(seed, 4)
    perm_s, perm_d = seed_key(seed, 5), seed_key(seed, 6)
    acc = KeyBuckets(n, ntup)
    for lo in range(0, ntup, chunk):
        e = torch.arange(lo, min(ntup, lo + chunk), dtype=torch.int64, device=device)
        ends = []
        for k, cw, pk in ((key_s, cum[0], perm_s), (key_d, cum[1], perm_d)):
            t = torch.remainder(_srl(rand64(k, e), 1), int(cw[-1]))
            idx = torch.searchsorted(cw, t, right=True)
            ends.append(feistel_permute(idx, n, pk))
        acc.add(ends[0], ends[1])
        del e, ends
    return acc.csr(name, device)


# --------------------------------------------------------------------------- #
# Named configurations (BASELINE.json configs)
# --------------------------------------------------------------------------- #
CONFIGS = {
    # C1: RMAT scale-16, ef 16 -- the parity config (oracle finishes in seconds)
    "C1": dict(kind="rmat", scale=16, edge_factor=16, seed=16),
    # C2: RMAT scale-22 (4M vertices, 67M edges) -- the N=1 bench workload
    "C2": dict(kind="rmat", scale=22, edge_factor=16, seed=22),
    # C3: LiveJournal-shaped Chung-Lu (4.8M vertices, ~69M edges)
    "C3": dict(kind="chunglu", n=4_800_000, m_target=69_000_000, alpha_out=1.9,
               dmax_out=20_000, alpha_in=2.0, dmax_in=14_000, oversample=1.03, seed=3),
    # C4: Twitter-shaped Chung-Lu (41.6M vertices, ~1.47B edges)
    "C4": dict(kind="chunglu", n=41_600_000, m_target=1_470_000_000, alpha_out=1.7,
               dmax_out=3_000_000, alpha_in=2.1, dmax_in=300_000, oversample=1.33, seed=41),
    # C5: RMAT scale-28 (268M vertices, 4.3B tuples)
    "C5": dict(kind="rmat", scale=28, edge_factor=16, seed=28),
    # small variants used by tests
    "T12": dict(kind="rmat", scale=12, edge_factor=16, seed=12),
    "T14": dict(kind="rmat", scale=14, edge_factor=16, seed=14),
    "LJ-small": dict(kind="chunglu", n=48_000, m_target=690_000, alpha_out=1.9,
                     dmax_out=2_000, alpha_in=2.0, dmax_in=1_400, oversample=1.06, seed=3),
}


def make(config: str, device="cpu", weights: bool = True, symmetric: bool = False,
         wmax: int = 64) -> Graph:
    """Build a named config's CSR (optionally with weights / symmetrised for CC)."""
    p = dict(CONFIGS[config])
    kind = p.pop("kind")
    seed = p["seed"]
    if kind == "rmat":
        g = rmat(p["scale"], p["edge_factor"], seed=seed, device=device, name=config)
    else:
        g = chung_lu(device=device, name=config, **p)
    if symmetric:
        g = symmetrize(g)
        g.name = config + "-sym"
    if weights:
        g = add_weights(g, seed ^ 0x5EED, wmax)
    return g


def first_source(g: Graph) -> int:
    """Reading R-7 ("the first source node"): smallest id with out-degree >= 1."""
    nz = torch.nonzero(g.degrees() > 0)
    return int(nz[0, 0]) if nz.numel() else 0


def sample_sources(g: Graph, count: int, seed: int) -> list:
    """``count`` distinct seeded vertices with out-degree >= 1 (R-7)."""
    cand = torch.nonzero(g.degrees() > 0).flatten()
    if cand.numel() == 0:
        return [0] * count
    h = rand64(seed_key(seed, 9), cand)
    order = torch.argsort(h)
    return [int(x) for x in cand[order[:count]].cpu()]
