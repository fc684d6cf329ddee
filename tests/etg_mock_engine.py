"""Test-only stand-in for the CUDA step engine: the same step interface
(begin / expand / scan / end, full-size labels and bitmap as torch int32
tensors) implemented with numpy on the CPU, so the multi-rank driver
(partitioning, exchange, termination) can be exercised with gloo here.
It is neither the oracle nor the product; results are checked against the oracle."""
import numpy as np
import torch

INF = 0xFFFFFFFF
CAP = 0xFFFFFFFE


class _Stats:
    def __init__(self):
        self.iterations = self.activations = self.frontier_total = self.shadows = self.edges_processed = 0


class MockEngine:
    def __init__(self, off, col, w, n):
        self.off = np.asarray(off, dtype=np.int64)
        self.col = np.asarray(col, dtype=np.int64)
        self.w = None if w is None else np.asarray(w, dtype=np.int64)
        self.n = n
        self.nwords = (n + 31) // 32
        self.q = torch.zeros(self.nwords, dtype=torch.int32)
        self.labels = torch.zeros(n, dtype=torch.int32)
        self.st = _Stats()

    def _lab(self):
        return self.labels.numpy().view(np.uint32)

    def _bits(self):
        return self.q.numpy().view(np.uint32)

    def begin(self, alg, source):
        self.alg, self.depth = alg, -1
        lab = self._lab()
        if alg == 2:
            lab[:] = np.arange(self.n, dtype=np.uint32)
            self._bits()[:] = 0
            for v in range(self.n):
                self._bits()[v >> 5] |= np.uint32(1 << (v & 31))
        else:
            lab[:] = 0 if alg == 3 else INF
            lab[source] = INF if alg == 3 else 0
            self._bits()[source >> 5] |= np.uint32(1 << (source & 31))
        self.st = _Stats()
        return self.scan()

    def scan(self):
        b = self._bits()
        act = [v for v in range(self.n) if (int(b[v >> 5]) >> (v & 31)) & 1]
        b[:] = 0
        self.depth += 1
        if self.alg == 0:
            self._lab()[act] = self.depth
        self.front = [v for v in act if self.off[v + 1] > self.off[v]]
        return len(act)

    def expand(self):
        lab = self._lab()
        src_lab = {v: int(lab[v]) for v in self.front}      # synchronous snapshot
        for v in self.front:
            for e in range(self.off[v], self.off[v + 1]):
                u = int(self.col[e])
                if self.alg == 0:
                    cand, better = self.depth + 1, lab[u] == INF
                elif self.alg == 1:
                    cand = min(src_lab[v] + int(self.w[e]), CAP)
                    better = cand < lab[u]
                elif self.alg == 2:
                    cand = src_lab[v]
                    better = cand < lab[u]
                else:
                    cand = min(src_lab[v], int(self.w[e]))
                    better = cand > lab[u]
                if better:
                    if self.alg != 0:
                        lab[u] = cand
                    self._bits()[u >> 5] |= np.uint32(1 << (u & 31))
                self.st.edges_processed += 1
        self.st.iterations += 1

    def end(self):
        return self.st
