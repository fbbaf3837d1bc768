"""bench.py's JSON-line contract (the driver parses it).

* CPU (-m "not gpu"): the reference arm (the oracle on host cores) prints one
  line with the keys the contract requires.
* GPU (-m gpu): a short run of the product arm on the small fp32 config
  prints one line with value / roofline / cpu_baseline / e2e / clocks /
  gpu_launches / dp_selfcheck, timing from >= 3 warm-up steps.
"""
import json
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
BASE_KEYS = {"metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better", "scaling",
             "vs_baseline", "dtype", "data", "config", "e2e", "cpu_baseline"}


def _line(args, timeout):
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py")] + args, capture_output=True, text=True,
                       timeout=timeout, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, r.stdout[-2000:]
    return json.loads(lines[0])


def test_reference_arm_line():
    d = _line(["--impl", "reference", "--config", "C1", "--steps", "1", "--warmup", "0"], 300)
    assert BASE_KEYS <= set(d) and d["impl"] == "reference"
    assert d["value"] > 0 and d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["cores"] >= 1
    assert d["e2e"]["h2d_bytes_per_step"] == 0 and d["higher_is_better"] is True


@pytest.mark.gpu
def test_product_arm_line():
    d = _line(["--config", "C1", "--steps", "20", "--warmup", "3", "--runs", "4", "--regions", "0",
               "--emulate-n", "0"], 900)
    assert BASE_KEYS <= set(d) and d["value"] > 0 and d["warmup"] >= 3
    for k in ("roofline", "clocks", "gpu_launches", "dp_selfcheck", "runs", "in_order"):
        assert k in d, k
    assert d["gpu_launches"] > 0 and d["dp_selfcheck"]["ok"] is True
    assert d["e2e"]["h2d_bytes_per_step"] > 0 and d["e2e"]["d2h_bytes_per_step"] > 0
    assert d["runs"]["n"] == 4 and abs(d["runs"]["mean_ms"] - d["ms_per_step"]) < 1e-9
    assert d["roofline"]["share_ok"] is True
