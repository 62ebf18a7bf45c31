"""bench.py's JSON contract on a real GPU (small sizes): one line with the driver's keys, the
roofline / cpu_baseline / e2e objects, and every parity flag true (the prefix sample and the
full-length segment certificate of the timed configuration)."""
import json
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _run(*args):
    out = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), *args], capture_output=True, text=True,
                         timeout=900, cwd=ROOT)
    assert out.returncode == 0, out.stderr[-3000:]
    lines = [l for l in out.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, out.stdout[-3000:]
    return json.loads(lines[0])


def test_default_config_line():
    d = _run("--size-gib", "1", "--steps", "3", "--warmup", "3")
    for key in ("metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better",
                "scaling", "vs_baseline", "dtype", "data", "config", "roofline", "clocks", "gpu_launches", "e2e",
                "cpu_baseline", "result"):
        assert key in d, key
    assert d["n_gpus"] == 1 and d["steps"] == 3 and d["warmup"] == 3 and d["value"] > 0
    r = d["roofline"]
    assert r["bound"] == "hbm" and r["peak"] > 0 and abs(r["frac"] - r["achieved"] / r["peak"]) < 1e-3
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["cores"] == 1
    assert d["e2e"]["h2d_bytes_per_step"] == d["config"]["input_bytes"]
    assert d["parity_sample"]["ok"] and d["parity_full"]["ok"]
    assert d["parity_full"]["bytes"] == d["config"]["input_bytes"]
    assert d["ablation"]["same_result"]
    assert d["gpu_launches"] >= d["steps"]


def test_tuned_html_line():
    d = _run("--config", "c4", "--size-gib", "0.25", "--steps", "3", "--warmup", "3", "--tune", "--no-e2e")
    assert d["tuning"]["k"] == 1 and d["tuning"]["candidates"] >= 3
    assert d["parity_sample"]["ok"] and d["ablation"]["same_result"]


def test_reference_arm_line():
    d = _run("--impl", "reference", "--size-gib", "0.05", "--steps", "1", "--warmup", "1")
    assert d["impl"] == "reference" and d["cpu_baseline"]["kind"] == "oracle" and d["value"] > 0
    assert d["e2e"]["h2d_bytes_per_step"] == 0
