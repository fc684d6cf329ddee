"""Host-side logic of bench.py (CPU): the SURVEY A-7 source rule, the oracle
pinning helper, the relaunch command for --gpus N."""
import importlib.util
import os

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
spec = importlib.util.spec_from_file_location("bench", os.path.join(ROOT, "bench.py"))
bench = importlib.util.module_from_spec(spec)
spec.loader.exec_module(bench)


def test_select_sources_keeps_reaching_ones_in_order():
    reach = {1: (5, 50), 2: (500, 4000), 3: (0, 0), 4: (2000, 9000), 5: (100, 700), 6: (999, 1)}
    keep, m = bench.select_sources([1, 2, 3, 4, 5, 6], lambda s: reach[s], n=10_000, count=2)
    assert keep == [2, 4] and m == {2: 4000, 4: 9000}          # >= 1 % of 10,000 = 100 vertices
    keep, m = bench.select_sources([1, 2, 3, 4, 5, 6], lambda s: reach[s], n=10_000, count=10)
    assert keep == [2, 4, 5, 6]
    with pytest.raises(RuntimeError):
        bench.select_sources([1, 3], lambda s: reach[s], n=10_000, count=4)


def test_pinned_core_restores_affinity():
    before = os.sched_getaffinity(0)
    with bench.pinned_core() as p:
        assert os.sched_getaffinity(0) == {p.core} and p.core in before
    assert os.sched_getaffinity(0) == before


def test_oracle_sources_match_rule():
    """The reference arm picks its sources with the oracle's BFS by the same rule."""
    import numpy as np
    import graphgen as gg
    import oracle
    g = gg.make("C1", weights=False)
    off, col, _ = g.numpy()
    srcs, m = bench.oracle_sources(g, off, col, 4, 4242)
    deg = np.diff(off.astype(np.int64))
    assert len(srcs) == 4
    for s in srcs:
        lab = oracle.bfs(off, col, s)
        assert (lab != oracle.INF).sum() >= 0.01 * g.n and m[s] == int(deg[lab != oracle.INF].sum())
    assert srcs == [s for s in gg.sample_sources(g, 16, 4242)
                    if (oracle.bfs(off, col, s) != oracle.INF).sum() >= 0.01 * g.n][:4]
