"""bench.py keeps its JSON contract (one line; the keys the driver and the judge
read), on the small C1 config so it runs in seconds."""
import json
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _run(*args):
    out = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), *args], cwd=ROOT,
                         capture_output=True, text=True, timeout=900)
    assert out.returncode == 0, out.stderr[-2000:]
    lines = [ln for ln in out.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1, out.stdout[-2000:]
    return json.loads(lines[0])


def test_bench_line_contract():
    d = _run("--config", "C1", "--steps", "2", "--warmup", "3", "--sources", "4")
    for k in ("metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better",
              "scaling", "vs_baseline", "dtype", "data", "config", "roofline", "cpu_baseline", "e2e",
              "gpu_launches", "clocks"):
        assert k in d, k
    assert d["unit"] == "GTEPS" and d["value"] > 0 and d["n_gpus"] == 1 and d["higher_is_better"] is True
    r = d["roofline"]
    for k in ("bound", "achieved", "peak", "unit", "frac", "traffic"):
        assert k in r, k
    assert 0 < r["frac"] < 1 and r["bound"] == "hbm"
    if r.get("l2"):                  # the L2-request roofline (committed ncu requests + measured ceiling)
        assert r["l2"]["achieved"] > 0 and r["l2"]["ceiling"] > 0 and 0 < r["l2"]["frac"] < 2
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["cores"] >= 1
    e = d["e2e"]
    assert e["value"] > 0 and e["h2d_bytes_per_step"] > 0 and e["d2h_bytes_per_step"] > 0
    assert d["gpu_launches"] > 0 and "workload" in d["config"]
    for k in ("sm_mhz", "sm_max_mhz", "reasons"):
        assert k in d["clocks"], k


def test_bench_reference_arm():
    d = _run("--impl", "reference", "--config", "C1", "--steps", "2", "--warmup", "3")
    assert d["impl"] == "reference" and d["value"] > 0 and d["cpu_baseline"]["kind"] == "oracle"
    assert d["e2e"]["h2d_bytes_per_step"] == 0


def test_bench_two_ranks_partitioned():
    """--gpus 2 without torchrun: bench.py relaunches itself with two ranks
    (here on one GPU), runs the partitioned path and rank 0 prints one line."""
    d = _run("--gpus", "2", "--config", "C1", "--steps", "2", "--warmup", "3", "--sources", "4", "--no-e2e")
    assert d["n_gpus"] == 2 and d["scaling"] == "strong" and d["value"] > 0
    assert "partition" in d["config"]["parallelism"] and d["gpu_launches"] > 0
