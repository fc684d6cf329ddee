"""GPU parity: the CUDA path through the C ABI vs the CPU oracle, bit-exact.

All labels are integers, and every result is a unique fixpoint (SURVEY 8(c)
"GPU = oracle"), so the bar is element-by-element equality of the n labels.
"""
import numpy as np
import pytest
import torch

import graphgen as gg
import oracle
from etg_testutil import load_golden, to_etg

pytestmark = pytest.mark.gpu

etg = pytest.importorskip("paper_conf_ipps_wangzlg19_b200")
U32 = etg.to_u32_numpy
INF = etg.INF


@pytest.fixture(scope="module", autouse=True)
def _built():
    from paper_conf_ipps_wangzlg19_b200 import _build
    _build.build()
    assert torch.cuda.is_available()


def check_all(g, sources, K=32, flags=0, algs=("bfs", "sssp", "sswp"), force_u64=False):
    off, col, w = g.numpy()
    G = to_etg(g, K=K, flags=flags, force_u64=force_u64)
    for s in sources:
        if "bfs" in algs:
            got, st = G.bfs(s)
            exp = oracle.bfs(off, col, s)
            np.testing.assert_array_equal(U32(got), exp, err_msg=f"BFS s={s} K={K} flags={flags}")
        if "sssp" in algs and w is not None:
            got, st = G.sssp(s)
            np.testing.assert_array_equal(U32(got), oracle.sssp(off, col, w, s),
                                          err_msg=f"SSSP s={s} K={K} flags={flags}")
        if "sswp" in algs and w is not None:
            got, st = G.sswp(s)
            np.testing.assert_array_equal(U32(got), oracle.sswp(off, col, w, s),
                                          err_msg=f"SSWP s={s} K={K} flags={flags}")
    return G


def check_cc(gs, K=32, flags=0):
    soff, scol, _ = gs.numpy()
    G = to_etg(gs, K=K, flags=flags, symmetric=True)
    got, st = G.cc()
    np.testing.assert_array_equal(U32(got), oracle.cc(soff, scol), err_msg=f"CC K={K} flags={flags}")
    return st


# --------------------------------------------------------------------------- #
# golden fixtures
# --------------------------------------------------------------------------- #
def _fixture_graph(f, key_w="w"):
    off = torch.tensor(f["off"], dtype=torch.int64)
    col = torch.tensor(f["col"], dtype=torch.int64)
    w = torch.tensor(f[key_w], dtype=torch.int64) if key_w in f else None
    return gg.Graph(f["id"], f["n"], off, col, w)


def test_golden_f1_bfs_udc_cc():
    f = load_golden("F1_fig3_udc.json")
    g = _fixture_graph(f)
    G = to_etg(g, K=f["K"])
    got, _ = G.bfs(f["bfs_source"])
    assert U32(got).tolist() == f["expect_bfs"]
    ids, st, en = G.udc_slices(torch.tensor(f["active"], device="cuda"))
    got = [[int(a), int(b), int(c)] for a, b, c in zip(U32(ids), st.cpu(), en.cpu())]
    assert got == f["expect_shadows"]                      # vertex 2 (degree 0) is filtered (L142)
    gs = gg.symmetrize(g)
    check_cc(gs, K=f["K"])


def test_golden_f2_f4():
    f = load_golden("F2_sssp_reactivation.json")
    G = to_etg(_fixture_graph(f))
    assert U32(G.bfs(f["source"])[0]).tolist() == f["expect_bfs"]
    assert U32(G.sssp(f["source"])[0]).tolist() == f["expect_sssp"]
    f = load_golden("F4_saturation.json")
    G = to_etg(_fixture_graph(f))
    assert U32(G.sssp(f["source"])[0]).tolist() == f["expect_sssp"]


def test_golden_f3_cc():
    f = load_golden("F3_cc_weak.json")
    g = gg.from_edges("F3", f["n"], f["edges"])
    gs = gg.symmetrize(g)
    G = to_etg(gs, symmetric=True)
    assert U32(G.cc()[0]).tolist() == f["expect_cc"]


# --------------------------------------------------------------------------- #
# C1 (the parity config) and the K / UDC / SMP / control sweeps
# --------------------------------------------------------------------------- #
@pytest.fixture(scope="module")
def c1():
    return gg.make("C1")


@pytest.fixture(scope="module")
def c1sym():
    return gg.make("C1", symmetric=True, weights=False)


def test_c1_all_algorithms(c1, c1sym):
    srcs = [gg.first_source(c1)] + gg.sample_sources(c1, 4, 11)
    check_all(c1, srcs)
    check_cc(c1sym)


@pytest.mark.parametrize("K", [1, 2, 3, 4, 10, 31, 32, 33, 64, 128, 1024])
def test_k_invariance(c1, c1sym, K):
    """Theorems 1-2 (L119-127): labels identical for every degree limit K."""
    srcs = gg.sample_sources(c1, 2, K)
    check_all(c1, srcs, K=K)
    check_cc(c1sym, K=K)
    if K <= 32:
        check_all(c1, srcs[:1], K=K, flags=128)      # shared-memory SMP stages


@pytest.mark.parametrize("flags", [2, 4, 32, 2 | 32, 4 | 32, 128, 128 | 32])
def test_flag_invariance(c1, c1sym, flags):
    """UDC off (L88 baseline), SMP off (Fig. 6 ablation: no look-ahead), shared-memory SMP,
    host-driven loop."""
    srcs = gg.sample_sources(c1, 2, 5)
    check_all(c1, srcs, flags=flags)
    check_cc(c1sym, flags=flags)


@pytest.mark.parametrize("tune", [64, 2, 2 | 64, 128])
def test_engine_variants(c1, c1sym, monkeypatch, tune):
    """Engine variants picked at load time (ETG_TUNE): 64 = SSSP/CC/SSWP commits mark the
    bitmap and the scan reads only it (no label/snapshot comparison);
    2 = the CTA-tile expand kernel; 128 = L2 bulk prefetch of the next tile's segments.
    Labels are the same unique fixpoints."""
    monkeypatch.setenv("ETG_TUNE", str(tune))
    srcs = gg.sample_sources(c1, 2, 17)
    check_all(c1, srcs)
    check_cc(c1sym)
    check_cc(c1sym, flags=32)


@pytest.mark.parametrize("env", [
    {"ETG_SCAN_LIST": "0"}, {"ETG_SCAN_LIST": "2"}, {"ETG_SCAN_ROWS": "0"}, {"ETG_SCAN_ROWS": "1"},
    {"ETG_SPLIT": "1"}, {"ETG_SPLIT": "2"}, {"ETG_PDL": "1"}, {"ETG_SCAN_KW": "32", "ETG_SCAN_LIST": "2"},
    {"ETG_AHEAD_MID": "0", "ETG_TUNE2": "1"}, {"ETG_DIRTY": "0"}, {"ETG_SCAN_KW": "32"},
    {"ETG_SCAN_KW": "32", "ETG_SCAN_LIST": "0"}])
def test_scan_and_split_modes(c1, c1sym, monkeypatch, env):
    """Load-time scan / expand modes: the vertex-list compaction (never / always),
    the bulk-copied offsets (off / from one active row), the tile split (off /
    2 warps), the programmatic expand -> scan edge, 32-row scan tiles on a small
    graph, the mid-size look-ahead and grab size, the dirty-row scans (which
    need 32-row scan warps: forced on the small graphs here).  A5 and A2 only reorder how the same active set is compacted and
    expanded, so labels stay the unique fixpoints; a hub whose
    shadows span many tiles and the skewed LJ-small shape exercise both paths."""
    for k, v in env.items():
        monkeypatch.setenv(k, v)
    check_all(c1, gg.sample_sources(c1, 2, 29))
    check_cc(c1sym)
    g = gg.make("LJ-small")
    check_all(g, gg.sample_sources(g, 1, 31), algs=("bfs", "sssp"))
    off, col, w = g.numpy()
    s = gg.sample_sources(g, 1, 37)[0]                  # the bench's SSSP schedule (wave, auto Delta)
    np.testing.assert_array_equal(U32(to_etg(g, sssp_delta="auto").sssp(s)[0]), oracle.sssp(off, col, w, s))
    n = 200_000
    hub = [(0, v) for v in range(1, 150_001)] + [(v, v + 1) for v in range(150_000, n - 1)]
    gh = gg.add_weights(gg.from_edges("hub", n, hub), 7)
    check_all(gh, [0, 150_000], algs=("bfs", "sssp"))


def test_u64_offsets(c1):
    check_all(c1, gg.sample_sources(c1, 2, 3), force_u64=True)


@pytest.mark.parametrize("env", [{}, {"ETG_SCAN_LIST": "2", "ETG_SCAN_ROWS": "1"}, {"ETG_SCAN_LIST": "0"}])
def test_u64_offsets_scan_paths(monkeypatch, env):
    """64-bit offsets through the scan's staged-offset and vertex-list paths
    (8-byte shared-memory offsets, 2 CTAs per SM) on the skewed LJ-small shape."""
    for k, v in env.items():
        monkeypatch.setenv(k, v)
    g = gg.make("LJ-small")
    check_all(g, gg.sample_sources(g, 2, 41), algs=("bfs", "sssp"), force_u64=True)


@pytest.mark.parametrize("cfg", ["T14", "LJ-small"])
def test_other_shapes(cfg):
    g = gg.make(cfg)
    check_all(g, gg.sample_sources(g, 3, 2))
    check_cc(gg.make(cfg, symmetric=True, weights=False))


# --------------------------------------------------------------------------- #
# edge cases
# --------------------------------------------------------------------------- #
def test_source_with_zero_outdegree(c1):
    deg = c1.degrees()
    s = int(torch.nonzero(deg == 0)[0, 0])
    G = to_etg(c1)
    got = U32(G.bfs(s)[0])
    assert got[s] == 0 and np.sum(got != INF) == 1
    assert U32(G.sswp(s)[0])[s] == INF


def test_tiny_and_empty_graphs():
    g = gg.from_edges("one", 1, [])
    G = to_etg(g)
    assert U32(G.bfs(0)[0]).tolist() == [0]
    g = gg.from_edges("two", 2, [(0, 1)], weights=[7])
    G = to_etg(g)
    assert U32(G.sssp(0)[0]).tolist() == [0, 7]
    assert U32(G.sssp(1)[0]).tolist() == [INF, 0]


def test_hub_spanning_many_tiles():
    """One hub with 300K out-edges: UDC cuts it into ~9.4K shadows over ~37 tiles."""
    n = 400_000
    hub = [(0, v) for v in range(1, 300_001)]
    tail = [(v, v + 1) for v in range(300_000, n - 1)]
    g = gg.add_weights(gg.from_edges("hub", n, hub + tail), 99)
    check_all(g, [0, 5, 300_000], algs=("bfs", "sssp"))
    check_all(g, [0], K=1, algs=("bfs",))


def test_in_degree_skew():
    """All edges into one vertex: heavy atomic contention on a single label."""
    n = 50_000
    e = [(v, 0) for v in range(1, n)] + [(0, v) for v in range(1, n, 7)]
    g = gg.add_weights(gg.from_edges("sink", n, e), 5)
    check_all(g, [1, 0], algs=("bfs", "sssp"))
    check_cc(gg.symmetrize(gg.from_edges("sink", n, e)))


def test_duplicates_and_self_loops_tolerated():
    e = [(0, 1), (0, 1), (1, 1), (1, 2), (2, 0), (2, 3), (2, 3)]
    g = gg.add_weights(gg.from_edges("dup", 5, e), 1)
    check_all(g, [0, 2])


def test_large_weights_saturate():
    n = 64
    e = [(i, i + 1) for i in range(n - 1)]
    g = gg.from_edges("sat", n, e, weights=[2**31 - 1] * (n - 1))
    check_all(g, [0], algs=("sssp",))


# --------------------------------------------------------------------------- #
# step A2 (UDC) through the library's own device mapping
# --------------------------------------------------------------------------- #
@pytest.mark.parametrize("K", [1, 4, 10, 32, 33, 1000])
def test_udc_slices_match_oracle(K):
    g = gg.make("LJ-small", weights=False)
    off, _, _ = g.numpy()
    deg = np.diff(off.astype(np.int64))
    cand = np.nonzero(deg > 0)[0]
    rng = np.random.default_rng(K)
    act = rng.choice(cand, size=5000, replace=False).astype(np.int64)
    act = np.concatenate([act, [int(np.argmax(deg))], np.nonzero(deg == 0)[0][:50]])
    G = to_etg(g, K=K)
    ids, st, en = G.udc_slices(torch.from_numpy(act).cuda())
    # the library keeps the active set as a bitmap: vertices in increasing id order
    eid, est, een = oracle.udc_slices(off, np.unique(act).astype(np.uint32), K)
    np.testing.assert_array_equal(U32(ids), eid)
    np.testing.assert_array_equal(st.cpu().numpy().astype(np.uint64), est)
    np.testing.assert_array_equal(en.cpu().numpy().astype(np.uint64), een)


# --------------------------------------------------------------------------- #
# statistics and the host-buffer entry
# --------------------------------------------------------------------------- #
def test_bfs_work_counters(c1):
    """L152: for BFS every reached vertex is active once; edges processed =
    m of the activatable subgraph; shadows = sum ceil(deg/K) over reached."""
    off, col, _ = c1.numpy()
    s = gg.first_source(c1)
    K = 16
    G = to_etg(c1, K=K)
    lab, st = G.bfs(s)
    exp = oracle.bfs(off, col, s)
    deg = np.diff(off.astype(np.int64))
    reached = exp != INF
    rs = G.reach_stats(lab)
    assert rs.vertices_reached == int(reached.sum())
    assert rs.edges_reached == int(deg[reached].sum())
    assert st.edges_processed == int(deg[reached].sum())
    assert st.shadows == int(((deg[reached] + K - 1) // K).sum())
    assert st.activations == int(reached.sum())          # every reached vertex is active once
    # the level-d active set is non-empty iff some depth-d vertex has out-edges
    assert st.iterations == int(exp[reached & (deg > 0)].max()) + 1


def test_run_host_matches(c1):
    off, col, w = c1.numpy()
    s = gg.first_source(c1)
    o = torch.from_numpy(off.astype(np.int64)).to(torch.int32).pin_memory()
    c = torch.from_numpy(col.view(np.int32)).pin_memory()
    ww = torch.from_numpy(w.view(np.int32)).pin_memory()
    out = torch.empty(c1.n, dtype=torch.int32).pin_memory()
    scratch = torch.empty(etg.host_scratch_bytes(c1.n, c1.m, True), dtype=torch.uint8, device="cuda")
    etg.run_host(etg.SSSP, o, c, ww, s, out, scratch)
    np.testing.assert_array_equal(out.numpy().view(np.uint32), oracle.sssp(off, col, w, s))
    etg.run_host(etg.BFS, o, c, None, s, out, scratch)
    np.testing.assert_array_equal(out.numpy().view(np.uint32), oracle.bfs(off, col, s))
    # the cached handle is reused for a DIFFERENT graph of the same n and m:
    # the result must follow the new CSR, and ETG_VALIDATE must check it
    col2 = ((col.astype(np.int64) + 1) % c1.n).astype(np.uint32)
    c2 = torch.from_numpy(col2.view(np.int32)).pin_memory()
    for _ in range(2):
        etg.run_host(etg.BFS, o, c2, None, s, out, scratch, flags=etg.VALIDATE)
        np.testing.assert_array_equal(out.numpy().view(np.uint32), oracle.bfs(off, col2, s))
    bad = c2.clone()
    bad[7] = c1.n + 3                                     # col >= n: same sizes, malformed
    with pytest.raises(etg.EtgError, match="EINVALID_CSR"):
        etg.run_host(etg.BFS, o, bad, None, s, out, scratch, flags=etg.VALIDATE)
    # CC only with an explicit symmetry assertion (no silent SYMMETRIC)
    with pytest.raises(etg.EtgError, match="ENOTSYM"):
        etg.run_host(etg.CC, o, c, None, 0, out, scratch)
    gs = gg.make("C1", symmetric=True, weights=False)
    soff, scol, _ = gs.numpy()
    so = torch.from_numpy(soff.astype(np.int64)).to(torch.int32).pin_memory()
    sc = torch.from_numpy(scol.view(np.int32)).pin_memory()
    scr = torch.empty(etg.host_scratch_bytes(gs.n, gs.m, False), dtype=torch.uint8, device="cuda")
    etg.run_host(etg.CC, so, sc, None, 0, out, scr, symmetric=True)
    np.testing.assert_array_equal(out.numpy().view(np.uint32), oracle.cc(soff, scol))


def test_errors():
    g = gg.from_edges("x", 3, [(0, 1)])
    G = to_etg(g)
    with pytest.raises(etg.EtgError, match="EINVAL"):
        G.bfs(5)
    with pytest.raises(etg.EtgError, match="ENOWEIGHTS"):
        G.sssp(0)
    with pytest.raises(etg.EtgError, match="ENOTSYM"):
        G.cc()
    bad = gg.Graph("bad", 3, torch.tensor([0, 1, 1, 1]), torch.tensor([7]))
    with pytest.raises(etg.EtgError, match="EINVALID_CSR"):
        to_etg(bad)


@pytest.mark.parametrize("delta", [1, 7, 16, 64, 1 << 20])
def test_sssp_near_far_schedule(c1, delta):
    """The near-far schedule defers far active vertices; distances are the same
    unique fixpoint (golden F2, saturation, C1, LJ-small, hub)."""
    off, col, w = c1.numpy()
    for s in gg.sample_sources(c1, 3, delta):
        G = to_etg(c1, sssp_delta=delta)
        np.testing.assert_array_equal(U32(G.sssp(s)[0]), oracle.sssp(off, col, w, s))
        Gh = to_etg(c1, sssp_delta=delta, flags=32)
        np.testing.assert_array_equal(U32(Gh.sssp(s)[0]), oracle.sssp(off, col, w, s))
    f = load_golden("F2_sssp_reactivation.json")
    G = to_etg(_fixture_graph(f), sssp_delta=delta)
    assert U32(G.sssp(f["source"])[0]).tolist() == f["expect_sssp"]
    f = load_golden("F4_saturation.json")
    G = to_etg(_fixture_graph(f), sssp_delta=delta)
    assert U32(G.sssp(f["source"])[0]).tolist() == f["expect_sssp"]
    g = gg.make("LJ-small")
    off, col, w = g.numpy()
    s = gg.first_source(g)
    np.testing.assert_array_equal(U32(to_etg(g, sssp_delta=delta).sssp(s)[0]), oracle.sssp(off, col, w, s))


def test_host_resident_edges(c1):
    """NEXT-2: col/w in pinned host memory, read zero-copy by the kernels."""
    off, col, w = c1.numpy()
    o, c, ww, fl = etg.csr_to_device(c1.off, c1.col, c1.w, device="cuda")
    ch, wh = c.cpu().pin_memory(), ww.cpu().pin_memory()
    G = etg.Graph(o, ch, wh, n=c1.n, flags=fl | etg.HOST_EDGES)
    for s in gg.sample_sources(c1, 2, 77):
        np.testing.assert_array_equal(U32(G.bfs(s)[0]), oracle.bfs(off, col, s))
        np.testing.assert_array_equal(U32(G.sssp(s)[0]), oracle.sssp(off, col, w, s))


def test_galois_gr_file_traversal(tmp_path, c1):
    """NEXT-4: a .gr file written from C1, read back, traversed on the GPU."""
    from paper_conf_ipps_wangzlg19_b200 import gr
    off, col, w = c1.numpy()
    p = str(tmp_path / "c1.gr")
    gr.write_gr(p, off.astype(np.int64), col, w)
    o2, c2, w2 = gr.read_gr(p)
    od, cd, wd, fl = etg.csr_to_device(torch.from_numpy(o2), torch.from_numpy(c2.astype(np.int64)),
                                       torch.from_numpy(w2.astype(np.int64)), device="cuda")
    G = etg.Graph(od, cd, wd, n=c1.n, flags=fl, validate=True)
    s = gg.first_source(c1)
    np.testing.assert_array_equal(U32(G.sssp(s)[0]), oracle.sssp(off, col, w, s))


@pytest.mark.parametrize("rows32", [False, True])
@pytest.mark.parametrize("classic", [False, True])
@pytest.mark.parametrize("delta", [3, 12, 40])
def test_sssp_wave_and_classic_near_far(c1, delta, classic, rows32, monkeypatch):
    """Both threshold rules of the near-far schedule: the wave (default: the
    threshold advances by Delta every iteration) and the classic one (advance
    only when the near set is empty; ETG_TUNE=8192).  Same distances.  rows32:
    32-row scan warps, so the dirty-row scans (rows marked by the sparse
    expands plus rows holding deferred vertices) run on these small graphs too."""
    monkeypatch.setenv("ETG_TUNE", "8192" if classic else "0")
    if rows32:
        monkeypatch.setenv("ETG_SCAN_KW", "32")
    off, col, w = c1.numpy()
    for s in gg.sample_sources(c1, 2, 100 + delta):
        G = to_etg(c1, sssp_delta=delta)
        d, st = G.sssp(s)
        np.testing.assert_array_equal(U32(d), oracle.sssp(off, col, w, s))
    g = gg.make("LJ-small", device="cuda")
    o2, c2_, w2 = g.to("cpu").numpy()
    s = gg.first_source(g)
    G = to_etg(g, sssp_delta=delta)
    np.testing.assert_array_equal(U32(G.sssp(s)[0]), oracle.sssp(o2, c2_, w2, s))


def test_sssp_delta_auto(c1):
    """ETG_SSSP_DELTA_AUTO: Delta from the mean weight, same distances; the
    step-wise API refuses it (ranks would each derive their own Delta)."""
    off, col, w = c1.numpy()
    G = to_etg(c1, sssp_delta="auto")
    for s in gg.sample_sources(c1, 2, 77):
        np.testing.assert_array_equal(U32(G.sssp(s)[0]), oracle.sssp(off, col, w, s))
    # the rule: Delta = 6 x mean weight / mean out-degree, rounded, at least 1
    assert G.sssp_delta() == max(1, int(6.0 * float(c1.w.double().mean()) / (c1.m / c1.n) + 0.5))
    # the step-wise API refuses a handle loaded with auto -- also after the
    # first SSSP resolved it (sticky): separately loaded partitions would each
    # derive their own Delta
    import ctypes
    lab = torch.empty(c1.n, dtype=torch.int32, device="cuda")
    na = ctypes.c_uint32()
    for h in (to_etg(c1, sssp_delta="auto"), G):
        assert etg.lib().etg_step_begin(h._h, etg.SSSP, 0, ctypes.c_void_p(lab.data_ptr()), ctypes.byref(na)) == -1
    # weights all 1: Delta = 6 x 1 / 16 -> 1 (at least 1), the wave then advances one hop per iteration
    g1 = gg.Graph("unit", c1.n, c1.off, c1.col, torch.ones_like(c1.w))
    o1, c1_, w1 = g1.numpy()
    s = gg.first_source(c1)
    np.testing.assert_array_equal(U32(to_etg(g1, sssp_delta="auto").sssp(s)[0]), oracle.bfs(o1, c1_, s))


def test_run_host_batch_matches(c1):
    """Several queries on one host graph (the CSR crosses the link once; weights
    arrive while BFS runs; labels go back while the next query runs)."""
    off, col, w = c1.numpy()
    o = torch.from_numpy(off.astype(np.int64)).to(torch.int32).pin_memory()
    c = torch.from_numpy(col.view(np.int32)).pin_memory()
    ww = torch.from_numpy(w.view(np.int32)).pin_memory()
    srcs = gg.sample_sources(c1, 3, 11)
    queries = [(etg.BFS, srcs[0]), (etg.SSSP, srcs[0]), (etg.SSWP, srcs[1]), (etg.BFS, srcs[2]),
               (etg.SSSP, srcs[2])]
    out = torch.empty(len(queries) * c1.n, dtype=torch.int32).pin_memory()
    scratch = torch.empty(etg.host_scratch_bytes(c1.n, c1.m, True), dtype=torch.uint8, device="cuda")
    for _ in range(2):                                   # the second call reuses the cached handle
        out.fill_(7)
        sts = etg.run_host_batch(queries, o, c, ww, out, scratch, sssp_delta="auto")
        got = out.numpy().view(np.uint32).reshape(len(queries), c1.n)
        fn = {etg.BFS: lambda s: oracle.bfs(off, col, s), etg.SSSP: lambda s: oracle.sssp(off, col, w, s),
              etg.SSWP: lambda s: oracle.sswp(off, col, w, s)}
        for k, (a, s) in enumerate(queries):
            np.testing.assert_array_equal(got[k], fn[a](s), err_msg=f"query {k}")
        assert len(sts) == len(queries) and all(st.iterations > 0 for st in sts)
    with pytest.raises(etg.EtgError, match="ENOWEIGHTS"):
        etg.run_host_batch(queries, o, c, None, out, scratch)
