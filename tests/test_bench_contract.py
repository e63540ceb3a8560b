"""bench.py's JSON line (the driver's contract) -- the reference arm runs on CPU."""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_reference_arm_json_line():
    out = subprocess.check_output([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference", "--config",
                                   "C1", "--steps", "1", "--warmup", "0", "--ref-sample-rows", "10000"],
                                  cwd=ROOT, timeout=300).decode().strip().splitlines()
    assert len(out) == 1
    d = json.loads(out[0])
    for k in ("metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better", "scaling",
              "vs_baseline", "dtype", "data", "config", "cpu_baseline", "e2e", "impl"):
        assert k in d, k
    assert d["impl"] == "reference" and d["value"] > 0 and d["unit"] == "rows/s"
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["cores"] == 1
    assert d["e2e"]["h2d_bytes_per_step"] == 0 and d["e2e"]["value"] == d["value"]
    assert "workload" in d["config"]


def test_reference_arm_split_rule():
    """--split reaches the reference arm: the oracle runs the same split rule (R26/R27)"""
    out = subprocess.check_output([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference", "--config",
                                   "C1", "--steps", "1", "--warmup", "0", "--ref-sample-rows", "10000", "--split", "2"],
                                  cwd=ROOT, timeout=300).decode().strip().splitlines()
    d = json.loads(out[-1])
    assert d["config"]["split"].startswith("k-means++") and d["value"] > 0
