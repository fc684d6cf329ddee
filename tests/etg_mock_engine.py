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
        self.snap = self._lab().copy()
        return self.scan()

    def scan(self):
        b = self._bits()
        act = set(v for v in range(self.n) if (int(b[v >> 5]) >> (v & 31)) & 1)
        if self.alg != 0:
            # SSSP/CC/SSWP: also every vertex whose label moved since its snapshot
            lab = self._lab()
            moved = np.nonzero(lab != self.snap)[0]
            act.update(int(v) for v in moved)
            self.snap[moved] = lab[moved]
        act = sorted(act)
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
                        q = self._owner(u)
                        if q is not None:               # fused push: the owner's copy too
                            pl = self.peers[q]
                            pl[u] = max(pl[u], cand) if self.alg == 3 else min(pl[u], cand)
                    self._bits()[u >> 5] |= np.uint32(1 << (u & 31))
                self.st.edges_processed += 1
        self.st.iterations += 1

    def end(self):
        return self.st

    # ---- push exchange (source partition) ----
    peers = None

    def set_peers(self, bounds, rank, peer_labels):
        """Loopback stand-in for peer memory: the other engines' label arrays."""
        self.pbounds, self.prank = list(bounds), rank
        self.peers = [t.numpy().view(np.uint32) for t in peer_labels]
        self.peered = len(bounds) > 2

    def _owner(self, u):
        if self.peers is None:
            return None
        q = int(np.searchsorted(np.asarray(self.pbounds), u, side="right")) - 1
        return None if q == self.prank else q

    def sync(self):
        pass

    def frontier(self):
        return len(self.front)

    def _moved_foreign(self, bounds, rank):
        lab = self._lab()
        own = np.zeros(self.n, dtype=bool)
        own[bounds[rank]:bounds[rank + 1]] = True
        return np.nonzero((lab != self.snap) & ~own)[0]

    def push_count(self, bounds, rank):
        mv = self._moved_foreign(bounds, rank)
        self._pb = (list(bounds), rank)
        return [int(((mv >= bounds[q]) & (mv < bounds[q + 1])).sum()) for q in range(len(bounds) - 1)]

    def push_pack(self, counts, rank):
        bounds, _ = self._pb
        mv = self._moved_foreign(bounds, rank)            # ascending = grouped by owner
        lab = self._lab()
        pairs = np.stack([mv.astype(np.uint32), lab[mv]], axis=1) if len(mv) else np.zeros((0, 2), np.uint32)
        self.snap[mv] = lab[mv]
        return torch.from_numpy(pairs.astype(np.uint32).view(np.int32).reshape(-1, 2).copy())

    def push_apply(self, pairs):
        lab = self._lab()
        pr = pairs.numpy().view(np.uint32).reshape(-1, 2)
        for u, val in pr:
            lab[u] = max(lab[u], val) if self.alg == 3 else min(lab[u], val)

    # ---- fused destination-partition exchange ----
    def set_dest_peers(self, bounds, rank, peer_q, peer_labels):
        """Loopback stand-in for peer memory: the other engines' bitmap / label tensors."""
        self.dbounds, self.drank = list(bounds), rank
        self.dpeer_q = [t.numpy().view(np.uint32) for t in peer_q]
        self.dpeer_l = [t.numpy().view(np.uint32) for t in peer_labels]
        self.dest_peered = True

    def publish(self):
        lo, hi = self.dbounds[self.drank], self.dbounds[self.drank + 1]
        for q in range(len(self.dbounds) - 1):
            if q == self.drank:
                continue
            if self.alg == 0:
                a, b = lo >> 5, (hi + 31) >> 5
                src = self._bits()[a:b]
                nz = np.nonzero(src)[0]
                self.dpeer_q[q][a + nz] = src[nz]
            else:
                lab = self._lab()
                mv = np.nonzero(lab[lo:hi] != self.snap[lo:hi])[0] + lo
                self.dpeer_l[q][mv] = lab[mv]
