"""Parity at the BASELINE sizes (VERDICT r1 "full-size parity"): the CUDA path
in the launch configuration bench.py times (device-resident trace, default
options, seed 12345) against the oracle ELEMENT BY ELEMENT on whole plans --
every cluster, every m_i, every sample row, the estimate and the bound.

* C5 (configs[4]): the whole 1e9-row trace when the host has the memory for
  the oracle (~32 GB: its sort records + the trace); otherwise the first 300M
  rows of C5 (all 10k kernels) for the whole plan, plus the ROOT leaves of
  every kernel above 3M rows of the full trace, each recomputed by the oracle
  on that kernel's rows (a kernel's leaves depend only on its rows).
* C4 (configs[3]) at its full 100M rows.
The inputs come from the CUDA generator (byte-identical to the numpy spec,
tests/test_gpu_parity.py::test_tracegen_cuda_matches_numpy); the oracle only
ever sees host copies of the trace, never GPU output."""
import numpy as np
import pytest

import oracle as O
import tracegen as G
from parity_util import Z95, assert_plans_equal

pytestmark = [pytest.mark.gpu, pytest.mark.slow]


@pytest.fixture(scope="module")
def ctx():
    import paper_conf_micro_chungnkk25_b200 as m
    m.build()
    c = m.Context(0)
    yield c
    c.close()


def _device_trace(name, n=None):
    import torch
    sp = G.spec(name, n=n)
    ds = G.DeviceSpec(sp, "cuda:0")
    kid = torch.empty(sp.n, dtype=torch.int32, device="cuda")
    tt = torch.empty(sp.n, dtype=torch.int32, device="cuda")
    G.generate_cuda(ds, kid, tt)
    torch.cuda.synchronize()
    return sp, kid, tt


def _host(x):
    return x.cpu().numpy().view(np.uint32)


def _avail_gb():
    import psutil
    return psutil.virtual_memory().available / 2 ** 30


@pytest.mark.timeout(3600)
def test_c5_full_plan_vs_oracle(ctx):
    import torch
    sp, kid, tt = _device_trace("C5")
    full = _avail_gb() >= 48
    got = ctx.plan(kid, tt, sp.n_kernels, eps=sp.eps, z=Z95, seed=12345)
    if full:
        hk, ht = _host(kid), _host(tt)
        del kid, tt
        torch.cuda.empty_cache()
        ref = O.plan(hk, ht, sp.n_kernels, eps=sp.eps, z=Z95, seed=12345)
        assert_plans_equal(got, ref)
        assert len(got["sample_row"]) == len(ref["sample_row"]) > 400_000
        return
    # not enough host memory for a 1e9-row oracle: the whole plan of a 300M-row
    # C5 prefix, and every big kernel of the full trace one by one
    cl = got["clusters"]
    counts = torch.bincount(kid, minlength=sp.n_kernels).cpu().numpy()
    for k in np.nonzero(counts > 3_000_000)[0]:
        sel = torch.nonzero(kid == int(k)).flatten()
        sub_t = _host(tt[sel])
        ref = O.plan(np.zeros(len(sub_t), np.uint32), sub_t, 1, eps=sp.eps, z=Z95, seed=12345)
        mine = cl[cl["kernel_id"] == k]
        for f in ("ordinal", "lo_ns", "hi_ns", "n", "sum_ns"):
            assert np.array_equal(mine[f].astype(np.int64), ref[f].astype(np.int64)), (k, f)
    del kid, tt
    sp, kid, tt = _device_trace("C5", n=300_000_000)
    got = ctx.plan(kid, tt, sp.n_kernels, eps=sp.eps, z=Z95, seed=12345)
    ref = O.plan(_host(kid), _host(tt), sp.n_kernels, eps=sp.eps, z=Z95, seed=12345)
    assert_plans_equal(got, ref)


@pytest.mark.timeout(1800)
@pytest.mark.parametrize("eps", [0.05, 0.01])
def test_c4_full_size_vs_oracle(ctx, eps):
    sp, kid, tt = _device_trace("C4")
    assert sp.n == 100_000_000
    got = ctx.plan(kid, tt, sp.n_kernels, eps=eps, z=Z95, seed=4)
    ref = O.plan(_host(kid), _host(tt), sp.n_kernels, eps=eps, z=Z95, seed=4)
    assert_plans_equal(got, ref)
