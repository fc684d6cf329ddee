"""Pins for the CPU oracle (oracle/oracle.c) against things other than itself.

Each pin is chosen so a plausible mistake in the oracle (dropped term, wrong
sign/index, transposed operand, missing saturation, direction not ignored in CC,
wrong slice bounds in UDC) fails at least one test:

* closed forms on hand-built graphs (path, star, clique, cycle, binary tree, grid,
  disjoint unions, isolated vertices, self-loops, duplicates);
* brute force on every small random graph: boolean matrix powers (BFS),
  exhaustive simple paths and Bellman-Ford (SSSP/SSWP), DFS (CC);
* independent library routines: scipy.sparse.csgraph and networkx;
* certificates that characterise the answer uniquely, on the C1 config;
* the golden fixtures under tests/golden/ (each cites its PAPER.md passage).
"""
import itertools
import math

import numpy as np
import pytest
import scipy.sparse as sp
import scipy.sparse.csgraph as csg

import graphgen as gg
import oracle
from etg_testutil import load_golden

INF, CAP = oracle.INF, oracle.CAP


def csr(n, edges, w=None, dedup=False):
    g = gg.from_edges("t", n, edges, weights=w, dedup=dedup)
    off, col, ww = g.numpy()
    return off, col, ww


def edges_of(off, col):
    src = np.repeat(np.arange(len(off) - 1), np.diff(off.astype(np.int64)))
    return src, col.astype(np.int64)


# --------------------------------------------------------------------------- #
# closed forms
# --------------------------------------------------------------------------- #
def test_bfs_path_star_clique_cycle():
    n = 10
    off, col, _ = csr(n, [(i, i + 1) for i in range(n - 1)])
    assert oracle.bfs(off, col, 0).tolist() == list(range(n))
    assert oracle.bfs(off, col, 4).tolist() == [INF] * 4 + list(range(6))
    star = [(0, i) for i in range(1, n)]
    off, col, _ = csr(n, star + [(i, 0) for i in range(1, n)])
    assert oracle.bfs(off, col, 0).tolist() == [0] + [1] * (n - 1)
    assert oracle.bfs(off, col, 3).tolist() == [1] + [2] * 2 + [0] + [2] * 6
    off, col, _ = csr(n, [(u, v) for u in range(n) for v in range(n) if u != v])
    assert oracle.bfs(off, col, 7).tolist() == [1] * 7 + [0] + [1] * 2
    off, col, _ = csr(n, [(i, (i + 1) % n) for i in range(n)])
    assert oracle.bfs(off, col, 3).tolist() == [(i - 3) % n for i in range(n)]


def test_bfs_binary_tree_and_grid():
    n = 63
    off, col, _ = csr(n, [(i, c) for i in range(n) for c in (2 * i + 1, 2 * i + 2) if c < n])
    assert oracle.bfs(off, col, 0).tolist() == [int(math.floor(math.log2(i + 1))) for i in range(n)]
    R, C = 7, 9
    idx = lambda r, c: r * C + c
    e = []
    for r in range(R):
        for c in range(C):
            for dr, dc in ((0, 1), (1, 0), (0, -1), (-1, 0)):
                if 0 <= r + dr < R and 0 <= c + dc < C:
                    e.append((idx(r, c), idx(r + dr, c + dc)))
    off, col, _ = csr(R * C, e)
    got = oracle.bfs(off, col, idx(2, 3))
    assert got.tolist() == [abs(r - 2) + abs(c - 3) for r in range(R) for c in range(C)]


def test_bfs_selfloop_duplicates_isolated():
    off, col, _ = csr(5, [(0, 0), (0, 1), (0, 1), (1, 2), (1, 2), (2, 2)])
    assert oracle.bfs(off, col, 0).tolist() == [0, 1, 2, INF, INF]
    off, col, _ = csr(3, [])
    assert oracle.bfs(off, col, 1).tolist() == [INF, 0, INF]


def test_sssp_closed_forms():
    w = [5, 1, 7, 3, 2]
    off, col, ww = csr(6, [(i, i + 1) for i in range(5)], w)
    assert oracle.sssp(off, col, ww, 0).tolist() == [0, 5, 6, 13, 16, 18]
    # complete graph with w(u,v) = |u - v|: dist(s, v) = |s - v| (triangle equality)
    n = 9
    E = [(u, v) for u in range(n) for v in range(n) if u != v]
    off, col, ww = csr(n, E, [abs(u - v) for u, v in E])
    for s in (0, 4, 8):
        assert oracle.sssp(off, col, ww, s).tolist() == [abs(s - v) for v in range(n)]
    # shortcut vs long path: the longer hop count must win when lighter
    off, col, ww = csr(4, [(0, 3), (0, 1), (1, 2), (2, 3)], [10, 1, 1, 1])
    assert oracle.sssp(off, col, ww, 0).tolist() == [0, 1, 2, 3]


def test_sssp_unit_weights_equals_bfs():
    g = gg.make("T12", weights=False)
    off, col, _ = g.numpy()
    ones = np.ones(col.shape[0], dtype=np.uint32)
    for s in gg.sample_sources(g, 3, 1):
        assert np.array_equal(oracle.sssp(off, col, ones, s), oracle.bfs(off, col, s))


def test_cc_closed_forms():
    # k disjoint directed cliques at offsets, plus isolated vertices
    blocks = [(2, 4), (7, 3), (11, 5)]
    E = []
    for b, k in blocks:
        E += [(b + i, b + j) for i in range(k) for j in range(k) if i != j]
    n = 16
    off, col, _ = csr(n, E)
    exp = list(range(n))
    for b, k in blocks:
        for i in range(k):
            exp[b + i] = b
    assert oracle.cc(off, col).tolist() == exp
    # direction must be ignored: a directed path pointing "down" still joins
    off, col, _ = csr(5, [(4, 3), (3, 2), (2, 1), (1, 0)])
    assert oracle.cc(off, col).tolist() == [0] * 5


def test_sswp_closed_forms():
    off, col, ww = csr(4, [(0, 1), (1, 2), (0, 2), (2, 3)], [5, 9, 3, 7])
    # widths: 1: 5 ; 2: max(min(5,9), 3) = 5 ; 3: min(5, 7) = 5
    assert oracle.sswp(off, col, ww, 0).tolist() == [INF, 5, 5, 5]
    off, col, ww = csr(3, [(0, 1)], [4])
    assert oracle.sswp(off, col, ww, 0).tolist() == [INF, 4, 0]


# --------------------------------------------------------------------------- #
# golden fixtures (tests/golden/*.json, each with its PAPER.md citation)
# --------------------------------------------------------------------------- #
def test_golden_f1_fig3():
    f = load_golden("F1_fig3_udc.json")
    off = np.array(f["off"], dtype=np.uint64)
    col = np.array(f["col"], dtype=np.uint32)
    assert oracle.bfs(off, col, f["bfs_source"]).tolist() == f["expect_bfs"]
    ids, st, en = oracle.udc_slices(off, f["active"], f["K"])
    got = [[int(a), int(b), int(c)] for a, b, c in zip(ids, st, en)]
    assert got == f["expect_shadows"]
    per = {str(v): int(np.sum(ids == v)) for v in f["active"]}
    assert per == f["expect_shadows_per_vertex"]
    full = [s for s in got if s[2] - s[1] == f["K"]]
    assert full == f["expect_full_shadows_smp"]
    src, dst = edges_of(off, col)
    soff, scol, _ = csr(f["n"], list(zip(src, dst)) + list(zip(dst, src)), dedup=True)
    assert oracle.cc(soff, scol).tolist() == f["expect_cc_symmetrised"]


def test_golden_f2_f3_f4():
    f = load_golden("F2_sssp_reactivation.json")
    off, col, w = (np.array(f[k], dtype=t) for k, t in (("off", np.uint64), ("col", np.uint32), ("w", np.uint32)))
    assert oracle.bfs(off, col, f["source"]).tolist() == f["expect_bfs"]
    assert oracle.sssp(off, col, w, f["source"]).tolist() == f["expect_sssp"]
    f = load_golden("F3_cc_weak.json")
    off, col, _ = csr(f["n"], f["edges"])
    assert oracle.cc(off, col).tolist() == f["expect_cc"]
    f = load_golden("F4_saturation.json")
    off, col, w = (np.array(f[k], dtype=t) for k, t in (("off", np.uint64), ("col", np.uint32), ("w", np.uint32)))
    assert oracle.sssp(off, col, w, f["source"]).tolist() == f["expect_sssp"]


# --------------------------------------------------------------------------- #
# brute force on tiny random graphs
# --------------------------------------------------------------------------- #
def random_graph(rng, n, p, wmax=20):
    E = [(u, v) for u in range(n) for v in range(n) if rng.random() < p]
    W = [int(rng.integers(1, wmax + 1)) for _ in E]
    return E, W


def all_simple_path_costs(n, E, W, s):
    adj = [[] for _ in range(n)]
    for (u, v), w in zip(E, W):
        adj[u].append((v, w))
    best_sum = [None] * n
    best_width = [None] * n

    def dfs(v, seen, tot, width):
        if best_sum[v] is None or tot < best_sum[v]:
            best_sum[v] = tot
        if best_width[v] is None or width > best_width[v]:
            best_width[v] = width
        for u, w in adj[v]:
            if u not in seen:
                seen.add(u)
                dfs(u, seen, tot + w, min(width, w))
                seen.remove(u)

    dfs(s, {s}, 0, INF)
    return best_sum, best_width


@pytest.mark.parametrize("seed", range(12))
def test_bruteforce_small(seed):
    rng = np.random.default_rng(seed)
    n = int(rng.integers(2, 8))
    E, W = random_graph(rng, n, float(rng.uniform(0.1, 0.6)))
    off, col, w = csr(n, E, W)
    if len(E):
        # csr() sorts edges: re-read the (edge, weight) pairs from the CSR
        src, dst = edges_of(off, col)
        E = list(zip(src.tolist(), dst.tolist()))
        W = w.tolist()
    A = np.zeros((n, n), dtype=bool)
    for u, v in E:
        A[u, v] = True
    for s in range(n):
        # BFS: depth = first power k with (e_s A^k)[v]
        exp = [INF] * n
        cur = np.zeros(n, dtype=bool)
        cur[s] = True
        for k in range(n):
            for v in np.nonzero(cur)[0]:
                if exp[v] == INF:
                    exp[v] = k
            cur = (cur.astype(np.int64) @ A.astype(np.int64)) > 0
        assert oracle.bfs(off, col, s).tolist() == exp
        best_sum, best_width = all_simple_path_costs(n, E, W, s)
        dist = [INF if b is None else min(b, CAP) for b in best_sum]
        assert oracle.sssp(off, col, w if len(E) else np.zeros(0, np.uint32), s).tolist() == dist
        # Bellman-Ford n-1 rounds agrees too
        bf = [INF] * n
        bf[s] = 0
        for _ in range(n - 1):
            for (u, v), ww in zip(E, W):
                if bf[u] != INF and bf[u] + ww < bf[v]:
                    bf[v] = bf[u] + ww
        assert bf == dist
        width = [0 if b is None else b for b in best_width]
        assert oracle.sswp(off, col, w if len(E) else np.zeros(0, np.uint32), s).tolist() == width
    # CC by DFS on the undirected version
    und = [[] for _ in range(n)]
    for u, v in E:
        und[u].append(v)
        und[v].append(u)
    lab = [None] * n
    for r in range(n):
        if lab[r] is None:
            stack = [r]
            lab[r] = r
            while stack:
                x = stack.pop()
                for y in und[x]:
                    if lab[y] is None:
                        lab[y] = r
                        stack.append(y)
    assert oracle.cc(off, col).tolist() == lab


def test_saturation_large_weights():
    rng = np.random.default_rng(5)
    n = 6
    E = [(i, i + 1) for i in range(n - 1)]
    W = [int(x) for x in rng.integers(2**30, 2**31, size=len(E))]
    off, col, w = csr(n, E, W)
    exp, tot = [0], 0
    for x in W:
        tot += x
        exp.append(min(tot, CAP))
    assert oracle.sssp(off, col, w, 0).tolist() == exp
    assert exp[-1] == CAP


# --------------------------------------------------------------------------- #
# library routines (scipy, networkx) on generator graphs
# --------------------------------------------------------------------------- #
def _to_scipy(off, col, w=None):
    n = len(off) - 1
    data = np.ones(len(col)) if w is None else w.astype(np.float64)
    return sp.csr_matrix((data, col.astype(np.int64), off.astype(np.int64)), shape=(n, n))


def _from_float(d):
    out = np.full(d.shape, INF, dtype=np.uint64)
    fin = np.isfinite(d)
    out[fin] = d[fin].astype(np.uint64)
    return out.astype(np.uint32)


@pytest.mark.parametrize("cfg", ["T12", "LJ-small"])
def test_scipy_bfs_sssp_cc(cfg):
    g = gg.make(cfg)
    off, col, w = g.numpy()
    M = _to_scipy(off, col)
    Mw = _to_scipy(off, col, w)
    for s in gg.sample_sources(g, 3, 7):
        d = csg.shortest_path(M, directed=True, unweighted=True, indices=s)
        assert np.array_equal(oracle.bfs(off, col, s), _from_float(d))
        d = csg.dijkstra(Mw, directed=True, indices=s)
        assert np.array_equal(oracle.sssp(off, col, w, s), _from_float(d))
    ncomp, lab = csg.connected_components(M, directed=True, connection="weak")
    got = oracle.cc(off, col)
    # canonicalise scipy's labels to the minimum member id
    first = np.full(ncomp, -1, dtype=np.int64)
    for v in range(len(lab)):
        if first[lab[v]] < 0:
            first[lab[v]] = v
    assert np.array_equal(got, first[lab].astype(np.uint32))
    assert len(np.unique(got)) == ncomp


def test_networkx_small():
    nx = pytest.importorskip("networkx")
    g = gg.make("T12")
    off, col, w = g.numpy()
    G = nx.DiGraph()
    G.add_nodes_from(range(g.n))
    src, dst = edges_of(off, col)
    G.add_weighted_edges_from(zip(src.tolist(), dst.tolist(), w.tolist()))
    s = gg.first_source(g)
    exp = np.full(g.n, INF, dtype=np.uint32)
    for v, d in nx.single_source_shortest_path_length(G, s).items():
        exp[v] = d
    assert np.array_equal(oracle.bfs(off, col, s), exp)
    exp = np.full(g.n, INF, dtype=np.uint32)
    for v, d in nx.single_source_dijkstra_path_length(G, s).items():
        exp[v] = d
    assert np.array_equal(oracle.sssp(off, col, w, s), exp)
    lab = np.empty(g.n, dtype=np.uint32)
    for comp in nx.weakly_connected_components(G):
        lab[list(comp)] = min(comp)
    assert np.array_equal(oracle.cc(off, col), lab)


# --------------------------------------------------------------------------- #
# certificates on the C1 parity config (unique characterisations)
# --------------------------------------------------------------------------- #
def bfs_certificate(off, col, s, d):
    src, dst = edges_of(off, col)
    d64 = d.astype(np.int64)
    assert d[s] == 0
    fin_u = d[src] != INF
    # no edge from a reached vertex to an unreached one, and d[v] <= d[u] + 1
    assert np.all(d[dst[fin_u]] != INF)
    assert np.all(d64[dst[fin_u]] <= d64[src[fin_u]] + 1)
    # every reached v != s has a tight in-edge
    tight = fin_u & (d64[dst] == d64[src] + 1)
    has = np.zeros(len(d), dtype=bool)
    has[dst[tight]] = True
    reached = d != INF
    reached[s] = False
    assert np.all(has[reached])


def sssp_certificate(off, col, w, s, d):
    src, dst = edges_of(off, col)
    d64 = d.astype(np.int64)
    assert d[s] == 0
    fin_u = d[src] != INF
    cand = np.minimum(d64[src] + w.astype(np.int64), CAP)
    assert np.all(d64[dst[fin_u]] <= cand[fin_u])
    tight = fin_u & (d64[dst] == cand)
    has = np.zeros(len(d), dtype=bool)
    has[dst[tight]] = True
    reached = d != INF
    reached[s] = False
    assert np.all(has[reached])


def cc_certificate(off, col, lab):
    src, dst = edges_of(off, col)
    assert np.all(lab[src] == lab[dst])
    v = np.arange(len(lab))
    assert np.all(lab <= v)
    assert np.all(lab[lab] == lab)


def test_certificates_c1():
    g = gg.make("C1")
    off, col, w = g.numpy()
    for s in [gg.first_source(g)] + gg.sample_sources(g, 2, 3):
        bfs_certificate(off, col, s, oracle.bfs(off, col, s))
        sssp_certificate(off, col, w, s, oracle.sssp(off, col, w, s))
    gs = gg.make("C1", symmetric=True, weights=False)
    soff, scol, _ = gs.numpy()
    lab = oracle.cc(soff, scol)
    cc_certificate(soff, scol, lab)
    ncomp = csg.connected_components(_to_scipy(soff, scol), directed=False)[0]
    assert len(np.unique(lab)) == ncomp


def test_certificate_rejects_wrong_answer():
    """The certificate itself must catch an off-by-one (guards the pin)."""
    g = gg.make("T12")
    off, col, w = g.numpy()
    s = gg.first_source(g)
    d = oracle.bfs(off, col, s).copy()
    v = int(np.nonzero((d != INF) & (d > 1))[0][0])
    d[v] += 1
    with pytest.raises(AssertionError):
        bfs_certificate(off, col, s, d)


# --------------------------------------------------------------------------- #
# UDC (Def. 3) oracle: closed form count, disjoint cover, bound K
# --------------------------------------------------------------------------- #
@pytest.mark.parametrize("K", [1, 2, 3, 4, 10, 31, 32, 33, 64, 1024, 1 << 40])
def test_udc_slices_properties(K):
    g = gg.make("LJ-small", weights=False)
    off, col, _ = g.numpy()
    deg = np.diff(off.astype(np.int64))
    act = np.array(gg.sample_sources(g, 200, K % 97) + [int(np.argmin(deg))], dtype=np.uint32)
    ids, st, en = oracle.udc_slices(off, act, K)
    d = deg[act.astype(np.int64)]
    assert len(ids) == int(np.sum((d + K - 1) // K))            # sum ceil(deg/K)
    assert np.all(en > st) and np.all(en - st <= K)
    pos = 0
    for v in act.tolist():                                        # disjoint, covering, in order
        b = int(off[v])
        while b < int(off[v + 1]):
            assert ids[pos] == v and st[pos] == b
            b = int(en[pos])
            pos += 1
        assert b == int(off[v + 1])
    assert pos == len(ids)
    # a shadow shorter than K is always the last of its vertex (SMP classes)
    short = np.nonzero(en - st < K)[0]
    assert np.all(en[short] == off[ids[short].astype(np.int64) + 1])


# --------------------------------------------------------------------------- #
# the device-side SSSP certificate used at C4 size (tests/etg_testutil.py) is
# itself pinned here, on CPU tensors: it accepts the oracle's distances and
# rejects every plausible wrong answer (SURVEY 8(c) O-SSSP certificate)
# --------------------------------------------------------------------------- #
@pytest.mark.parametrize("cfg", ["C1", "LJ-small"])
def test_sssp_certificate_gpu_pinned(cfg):
    import torch
    from etg_testutil import sssp_certificate_gpu
    g = gg.make(cfg)
    off, col, w = g.numpy()
    for s in [gg.first_source(g)] + gg.sample_sources(g, 1, 5):
        d = oracle.sssp(off, col, w, s)
        ok = torch.from_numpy(d.astype(np.int64))
        assert sssp_certificate_gpu(g, s, ok, chunk=1 << 18) is None
        reached = np.nonzero((d != INF) & (d > 0))[0]
        unreached = np.nonzero(d == INF)[0]
        rng = np.random.default_rng(s)
        bad = []
        for v in rng.choice(reached, 3, replace=False):
            for delta in (+1, -1):                        # off by one either way
                x = d.astype(np.int64).copy()
                x[v] += delta
                bad.append(x)
        x = d.astype(np.int64).copy()
        x[s] = 1                                          # source not at 0
        bad.append(x)
        x = d.astype(np.int64).copy()
        x[reached[0]] = INF                               # a reached vertex reported unreached
        bad.append(x)
        if unreached.size:
            x = d.astype(np.int64).copy()
            x[unreached[0]] = int(d[reached].max())       # an unreached vertex reported reached
            bad.append(x)
        for x in bad:
            assert sssp_certificate_gpu(g, s, torch.from_numpy(x), chunk=1 << 18) is not None
