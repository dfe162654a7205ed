"""The bench.py JSON contract (the driver parses one line per run).

CPU: the reference arm (the oracle on the host) at config 1 size.
GPU: our arm at a small N with every block of the default line."""
import json
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _run(args, timeout=600):
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), *args], capture_output=True, text=True,
                       timeout=timeout, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [ln for ln in r.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1, r.stdout
    return json.loads(lines[0])


def test_metric_names():
    sys.path.insert(0, ROOT)
    import bench
    assert bench.metric_name({"theta": 0.5, "n": 10_000_000}) == "BH step bodies/s (theta=0.5, N=10M)"
    assert bench.metric_name({"theta": 0.3, "n": 1024}) == "BH step bodies/s (theta=0.3, N=1024)"
    assert bench.n_str(100_000_000) == "100M" and bench.n_str(1_000_000) == "1M"


def test_reference_arm_line():
    d = _run(["--impl", "reference", "--config", "cfg1", "--steps", "2", "--warmup", "0", "--cpu-seconds", "0.3"])
    assert d["impl"] == "reference" and d["unit"] == "bodies/s" and d["higher_is_better"] is True
    assert d["metric"] == "BH step bodies/s (theta=0.5, N=1024)"
    assert d["value"] > 0 and d["ms_per_step"] > 0 and d["steps"] == 2
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["cores"] >= 1
    assert d["e2e"]["h2d_bytes_per_step"] == 0 and d["e2e"]["value"] == d["value"]


@pytest.mark.gpu
def test_our_arm_line():
    d = _run(["--n", "200000", "--steps", "3", "--warmup", "3", "--no-cpu-baseline", "--repeats", "3"])
    assert d["impl"] == "ours" and d["n_gpus"] == 1 and d["steps"] == 3 and d["warmup"] == 3
    assert d["value"] > 0 and abs(d["value"] - 200000 / (d["ms_per_step"] / 1e3)) < 1e-6 * d["value"]
    assert len(d["repeats_ms"]) == 3
    r = d["roofline"]
    assert r["bound"] == "alu" and 0 < r["frac"] < 1 and r["peak"] > 0 and r["achieved"] > 0
    assert d["e2e"]["h2d_bytes_per_step"] == 28 * 200000 and d["e2e"]["d2h_bytes_per_step"] == 12 * 200000
    assert d["gpu_launches"] > 0 and "sm_mhz" in d["clocks"]
    assert d["interactions_per_s"] > 0
