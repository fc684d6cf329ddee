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


def test_l2_roofline_from_traffic_and_ceiling(tmp_path, monkeypatch):
    """The L2-request roofline object: requests per launch (ncu) over the bench's
    mean launch time, against the committed random-request ceiling; absent when
    either input is missing."""
    import json
    assert bench.l2_roofline(None, None, 0.1) is None
    assert bench.l2_roofline({"launches": 3}, "x.json", 0.1) is None          # capture without L2 counts
    (tmp_path / "profiles" / "r03").mkdir(parents=True)
    (tmp_path / "profiles" / "r03" / "l2_ceiling.json").write_text(
        json.dumps({"ceiling_g_per_s": 250.0, "source": "test"}))
    monkeypatch.setattr(bench, "ROOT", str(tmp_path))
    tr = {"l2_requests_per_launch": 25e6, "l2_requests_per_edge": 1.25}
    r = bench.l2_roofline(tr, "t.json", 0.2)                                  # 25 M requests in 0.2 ms
    assert r["achieved"] == pytest.approx(125.0) and r["ceiling"] == 250.0 and r["frac"] == pytest.approx(0.5)
    assert r["requests_per_edge"] == 1.25 and "t.json" in r["source"]


def test_traffic_summary_l2_fields(tmp_path):
    """tools/traffic_summary.py: dram and L2 request totals of the expand launches
    against the algorithmic bytes of the same calls (SURVEY 8(d) bytes model)."""
    import json
    import subprocess
    import sys
    rows = ['"ID","Kernel Name","Metric Name","Metric Unit","Metric Value"']
    for i in range(2):
        for name, unit, val in (("gpu__time_duration.sum", "usecond", "100"), ("dram__bytes_read.sum", "Mbyte", "8"),
                                ("dram__bytes_write.sum", "byte", "0"),
                                ("lts__t_requests_srcunit_tex.sum", "", "1,000,000"),
                                ("lts__t_sectors_srcunit_tex.sum", "sector", "3000000")):
            rows.append(f'"{i}","expand_warp_kernel","{name}","{unit}","{val}"')
    (tmp_path / "l.csv").write_text("\n".join(rows) + "\n")
    stats = {"config": "T", "calls": [{"alg": "bfs", "edges_processed": 1_000_000, "frontier_total": 1000}]}
    (tmp_path / "s.json").write_text(json.dumps(stats))
    out = subprocess.run([sys.executable, os.path.join(ROOT, "tools", "traffic_summary.py"),
                          str(tmp_path / "l.csv"), str(tmp_path / "s.json")], capture_output=True, text=True)
    d = json.loads(out.stdout)
    assert d["launches"] == 2 and d["alg_bytes_total"] == 8 * 1_000_000 + 20 * 1000
    assert d["dram_bytes_total"] == 16e6 and d["l2_requests_total"] == 2e6
    assert d["l2_requests_per_launch"] == 1e6 and d["l2_requests_per_edge"] == 2.0
    assert d["l2_g_requests_per_s_under_ncu"] == pytest.approx(2e6 / 200e-6 / 1e9)
