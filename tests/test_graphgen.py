"""The shared input generators: determinism, exact integer arithmetic, shape."""
import numpy as np
import pytest
import torch

import graphgen as gg


def test_rand64_matches_numpy_uint64():
    ctr = np.arange(0, 1 << 16, dtype=np.int64) * 7919 + 3
    for seed in (0, 1, 22, 2**40 + 5):
        key = gg.seed_key(seed, 1)
        a = gg.rand64(key, torch.from_numpy(ctr)).numpy().view(np.uint64)
        b = gg.rand64_numpy(key, ctr)
        assert np.array_equal(a, b)


def test_splitmix64_known_value():
    # SplitMix64 reference stream for seed 0: first output 0xE220A8397B1DCDAF
    z = gg.mix64(torch.tensor([gg._s64(gg.GAMMA)], dtype=torch.int64)).numpy().view(np.uint64)
    assert int(z[0]) == 0xE220A8397B1DCDAF


@pytest.mark.parametrize("n", [1, 2, 5, 64, 1000, 4097])
def test_feistel_is_bijection(n):
    x = torch.arange(n, dtype=torch.int64)
    y = gg.feistel_permute(x, n, gg.seed_key(3, 2))
    assert sorted(y.tolist()) == list(range(n))


def test_rmat_deterministic_and_clean():
    a = gg.make("T12")
    b = gg.make("T12")
    assert a.sha256() == b.sha256()
    off, col, w = a.numpy()
    src = np.repeat(np.arange(a.n), np.diff(off.astype(np.int64)))
    assert np.all(src != col)                                   # no self-loops
    key = src.astype(np.int64) * a.n + col
    assert np.all(np.diff(key) > 0)                             # sorted, no duplicates
    assert w.min() >= 1 and w.max() <= 64
    assert gg.make("T12", weights=True).sha256() != gg.make("T14").sha256()


def test_rmat_c1_shape():
    """C1 shape targets: m_dedup ~ 1.044M, ~10% zero out-degree."""
    g = gg.make("C1", weights=False)
    deg = g.degrees()
    assert g.n == 65536
    assert 1_000_000 < g.m < 1_048_576
    assert 0.07 < float((deg == 0).float().mean()) < 0.13
    assert 800 < int(deg.max()) < 4000


def test_chunglu_small_shape():
    g = gg.make("LJ-small", weights=False)
    deg = g.degrees()
    assert 600_000 < g.m < 760_000
    assert int(deg.max()) > 500


def test_weights_are_function_of_endpoints():
    g = gg.make("T12")
    s = gg.symmetrize(gg.make("T12", weights=False))
    s = gg.add_weights(s, 12 ^ 0x5EED)
    # an edge present in both graphs gets the same weight
    off, col, w = g.numpy()
    soff, scol, sw = s.numpy()
    v = gg.first_source(g)
    for e in range(int(off[v]), int(off[v + 1])):
        u = col[e]
        k = np.searchsorted(scol[int(soff[v]):int(soff[v + 1])], u)
        assert sw[int(soff[v]) + k] == w[e]


def test_symmetrize():
    g = gg.from_edges("t", 4, [(0, 1), (1, 2), (3, 3)])
    s = gg.symmetrize(g)
    off, col, _ = s.numpy()
    assert off.tolist() == [0, 1, 3, 4, 4]
    assert col.tolist() == [1, 0, 2, 1]


def test_bucketed_dedup_is_equivalent(monkeypatch):
    """Large graphs are deduplicated per source-range bucket: same CSR."""
    a = gg.make("T12")
    monkeypatch.setattr(gg, "_BUCKET_TUPLES", 1 << 10)
    b = gg.make("T12")
    assert a.sha256() == b.sha256()
    c = gg.make("LJ-small", weights=False)
    monkeypatch.setattr(gg, "_BUCKET_TUPLES", 1 << 27)
    d = gg.make("LJ-small", weights=False)
    assert c.sha256() == d.sha256()


def test_galois_gr_roundtrip(tmp_path):
    """NEXT-4: the .gr reader/writer round-trips CSR + weights, v1 and v2."""
    from paper_conf_ipps_wangzlg19_b200 import gr
    g = gg.make("T12")
    off, col, w = g.numpy()
    for version in (1, 2):
        for weights in (None, w):
            p = str(tmp_path / f"g{version}{weights is None}.gr")
            gr.write_gr(p, off.astype(np.int64), col, weights, version=version)
            o2, c2, w2 = gr.read_gr(p)
            assert np.array_equal(o2, off.astype(np.int64)) and np.array_equal(c2, col)
            assert (w2 is None) == (weights is None)
            if weights is not None:
                assert np.array_equal(w2, w)
    odd = gg.from_edges("odd", 3, [(0, 1), (1, 2), (2, 0)])
    o, c, _ = odd.numpy()
    p = str(tmp_path / "odd.gr")
    gr.write_gr(p, o.astype(np.int64), c)                 # m odd: v1 pads to 8 bytes
    assert np.array_equal(gr.read_gr(p)[1], c)
    with open(p, "r+b") as f:                               # corrupt the size
        f.truncate(40)
    with pytest.raises(ValueError):
        gr.read_gr(p)


def _golden_sha():
    import json
    import os
    return json.load(open(os.path.join(os.path.dirname(__file__), "golden", "config_sha256.json")))


@pytest.mark.parametrize("cfg", ["T12", "C1", "LJ-small"])
def test_config_sha256_pinned(cfg):
    """Input provenance: the CSR of each small config is pinned by
    its SHA-256 (tests/golden/config_sha256.json, written by tools/config_sha.py)."""
    gold = _golden_sha()
    g = gg.make(cfg)
    assert gold[cfg + "+w"] == {"n": g.n, "m": g.m, "sha256": g.sha256()}
    s = gg.make(cfg, symmetric=True, weights=False)
    assert gold[cfg + "-sym"] == {"n": s.n, "m": s.m, "sha256": s.sha256()}


@pytest.mark.gpu
@pytest.mark.parametrize("cfg", ["T14", "C1", "LJ-small"])
def test_generator_cpu_equals_cuda(cfg):
    """The same integer arithmetic on the GPU gives the same graphs, bit for bit
    (graphgen module doc): CUDA-built CSR = the CPU-built one = the pinned hash."""
    gold = _golden_sha()
    for sym in (False, True):
        gc = gg.make(cfg, device="cpu", symmetric=sym, weights=not sym)
        gd = gg.make(cfg, device="cuda", symmetric=sym, weights=not sym)
        assert torch.equal(gc.off, gd.off.cpu()) and torch.equal(gc.col, gd.col.cpu())
        assert (gc.w is None) == (gd.w is None) and (gc.w is None or torch.equal(gc.w, gd.w.cpu()))
        assert gd.sha256() == gold[cfg + ("-sym" if sym else "+w")]["sha256"]
