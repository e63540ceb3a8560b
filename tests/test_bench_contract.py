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


def test_gpus_flag_launches_ranks_reference_arm():
    """--gpus N without a torchrun environment re-execs bench.py under torchrun
    with N ranks (127.0.0.1 rendezvous); rank 0 alone prints the reference line,
    which reports the rank count (CPU-only: the reference arm needs no GPU)."""
    out = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference", "--config", "C1",
                          "--gpus", "2", "--steps", "1", "--warmup", "0", "--ref-sample-rows", "5000"],
                         cwd=ROOT, timeout=600, capture_output=True, text=True)
    assert out.returncode == 0, out.stderr[-2000:]
    lines = [l for l in out.stdout.strip().splitlines() if l.startswith("{")]
    assert len(lines) == 1, out.stdout
    d = json.loads(lines[0])
    assert d["n_gpus"] == 2 and d["impl"] == "reference"


def test_gpus_flag_fails_loudly_without_devices():
    """our arm never silently runs on fewer GPUs than --gpus asks for"""
    import torch
    if torch.cuda.device_count() >= 2:
        import pytest
        pytest.skip("enough GPUs here")
    out = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", "2", "--steps", "1"], cwd=ROOT,
                         timeout=300, capture_output=True, text=True)
    assert out.returncode != 0
    assert "CUDA devices" in out.stdout


def test_gpus_flag_dry_launch_and_world_mismatch():
    out = subprocess.check_output([sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", "8", "--dry-launch"],
                                  cwd=ROOT, timeout=300).decode()
    cmd = json.loads(out.strip().splitlines()[-1])["launch"]
    assert "torch.distributed.run" in cmd and "--nproc-per-node=8" in cmd and "--master-addr=127.0.0.1" in cmd
    assert cmd[-4:] == ["--gpus", "8"] or "--gpus" in cmd
    env = dict(os.environ, WORLD_SIZE="2", RANK="0", LOCAL_RANK="0")
    out = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", "4", "--impl", "reference"],
                         cwd=ROOT, timeout=300, capture_output=True, text=True, env=env)
    assert out.returncode != 0 and "WORLD_SIZE=2" in out.stdout
