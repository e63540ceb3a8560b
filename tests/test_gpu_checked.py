"""Bounds-checked build (the stand-in for compute-sanitizer's memcheck, which
the GPU pool has disabled): the library compiled with -DSR_CHECK traps on any
out-of-range index at the checked sites (SR_DCHECK in common.cuh: the sort's
scatter and write-out, the split descent's stack and chunk ranges, the decide
kernel's frontier appends, the sampler's positions and ambiguous-sample list).
Every path of tools/sanitize_run.py (three split rules, metric bounds, host
pointers, census, scopes, a 2-rank loopback plan) and a 100M-row C5-shaped
bench plan must run to completion under it."""
import json
import os
import subprocess
import sys

import pytest

pytestmark = [pytest.mark.gpu, pytest.mark.slow]
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
LIB = os.path.join(ROOT, "paper_conf_micro_chungnkk25_b200", "lib", "libstemroot_check.so")


@pytest.fixture(scope="module")
def env():
    e = dict(os.environ, SR_EXTRA_NVCC="-DSR_CHECK", STEMROOT_LIB=LIB)
    subprocess.run([sys.executable, "-c", "import paper_conf_micro_chungnkk25_b200 as m; m.build()"], env=e,
                   check=True, cwd=ROOT, timeout=1200)
    return e


@pytest.mark.timeout(1800)
@pytest.mark.parametrize("cfg", ["C1", "C2"])
def test_checked_build_every_path(env, cfg):
    out = subprocess.run([sys.executable, os.path.join(ROOT, "tools", "sanitize_run.py"), cfg], env=env,
                         capture_output=True, text=True, timeout=1500, cwd=ROOT)
    log = out.stdout + out.stderr
    assert "SR_CHECK failed" not in log, log[-4000:]
    assert out.returncode == 0 and "SANITIZE_RUN_OK" in log, log[-4000:]


@pytest.mark.timeout(1800)
def test_checked_build_bench_size(env):
    out = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--n", "100000000", "--steps", "1",
                          "--warmup", "0", "--no-e2e", "--no-cpu-baseline"], env=env, capture_output=True, text=True,
                         timeout=1500, cwd=ROOT)
    log = out.stdout + out.stderr
    assert "SR_CHECK failed" not in log, log[-4000:]
    assert out.returncode == 0, log[-4000:]
    line = json.loads(out.stdout.strip().splitlines()[-1])
    assert line["config"]["clusters"] > 0 and line["config"]["samples"] > 0
