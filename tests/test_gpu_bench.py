"""bench.py's JSON line (the driver's contract) on a small configuration: one line, the contract keys, the
SURVEY 8(d) roofline recomputed from its own fields, an end-to-end leg with declared copies, and a
reference arm line for the same metric."""
import json
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _run(*args):
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), *args], capture_output=True, text=True,
                       cwd=ROOT, timeout=600)
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [ln for ln in r.stdout.splitlines() if ln.strip()]
    assert len(lines) == 1, r.stdout
    return json.loads(lines[0])


@pytest.mark.gpu
def test_bench_line_contract_small_config():
    d = _run("--config", "1", "--steps", "3", "--warmup", "3", "--e2e-steps", "1", "--no-cpu-baseline",
             "--steady-chunks", "0")
    for k in ("metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better", "scaling",
              "vs_baseline", "dtype", "data", "config", "roofline", "e2e", "gpu_launches", "clocks", "kernels",
              "phases_ms_per_step", "breakdown"):
        assert k in d, k
    assert d["n_gpus"] == 1 and d["steps"] == 3 and d["warmup"] == 3 and d["higher_is_better"] is True
    assert d["value"] > 0 and d["ms_per_step"] > 0 and d["gpu_launches"] > 0
    rf = d["roofline"]
    # frac = B_min / step time / peak, from the line's own numbers
    want = rf["bytes_min"] / (d["ms_per_step"] / 1e3) / 1e9 / rf["peak"]
    assert abs(rf["frac"] - want) < 1e-6 * max(1.0, want)
    e = d["e2e"]
    assert e["value"] > 0 and e["h2d_bytes_per_step"] > 0 and e["d2h_bytes_per_step"] > 0


@pytest.mark.gpu
def test_reference_arm_line():
    d = _run("--impl", "reference", "--config", "1", "--steps", "1", "--warmup", "1")
    assert d["impl"] == "reference" and d["value"] > 0
    assert d["e2e"]["h2d_bytes_per_step"] == 0 and d["e2e"]["d2h_bytes_per_step"] == 0
    assert d["cpu_baseline"]["kind"] == "oracle"
