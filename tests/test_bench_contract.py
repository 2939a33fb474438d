"""bench.py's JSON line (the driver's contract): the reference arm on CPU (the
oracle, this tier's reference), our arm on the GPU (-m gpu).  Each runs the
real script in a subprocess and checks the keys, types and internal
consistency of its single JSON line."""
import json
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
METRIC = "Boids agent-steps/sec at 1/2/4/8 B200; % FP32 peak (search), % HBM BW (update)"


def _run(*args, timeout=600):
    out = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), *args], cwd=ROOT, capture_output=True,
                         text=True, timeout=timeout)
    assert out.returncode == 0, out.stderr[-2000:]
    lines = [ln for ln in out.stdout.splitlines() if ln.strip()]
    assert len(lines) == 1, out.stdout  # exactly one JSON line
    return json.loads(lines[0])


def _common(d, workload):
    assert d["metric"] == METRIC and d["unit"] == "agent-steps/s"
    assert d["higher_is_better"] is True and d["n_gpus"] == 1
    assert d["value"] > 0 and d["ms_per_step"] > 0
    assert d["config"]["workload"] == workload and d["data"] == "synthetic"
    assert d["vs_baseline"] is None  # BASELINE.md holds no published number for this metric


def test_reference_arm_line():
    d = _run("--impl", "reference", "--workload", "c1", "--steps", "3", "--warmup", "3")
    _common(d, "c1")
    assert d["impl"] == "reference"
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["value"] == d["value"]
    assert d["e2e"] == {"value": d["value"], "unit": d["unit"], "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}


@pytest.mark.gpu
def test_gpu_arm_line_matches_reference_config():
    d = _run("--workload", "c1", "--steps", "3", "--warmup", "3", timeout=900)
    _common(d, "c1")
    ref = _run("--impl", "reference", "--workload", "c1", "--steps", "3", "--warmup", "3")
    assert d["config"] == ref["config"]  # the driver compares the two arms on the same config
    r = d["roofline"]
    assert r["bound"] == "alu" and 0 < r["frac"] < 1.5 and r["peak"] > 0 and r["achieved"] > 0
    assert "k_small" in r["kernel"]  # n = 1024: the one-kernel warm step
    assert d["gpu_launches"] >= 3 and d["dtype"] == "f32"
    e = d["e2e"]
    assert e["value"] > 0 and e["h2d_bytes_per_step"] == 1024 * 13 * 4 == e["d2h_bytes_per_step"]
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["cores"] == 1
    c = d["clocks"]
    assert c["sm_mhz"] > 0 and isinstance(c["reasons"], list)
    assert d["update_roofline"]["bound"] == "hbm" and d["update_roofline"]["frac"] > 0
