"""Host-side logic of the multi-GPU path with world_size 2 on CPU (gloo):
kernel-id owner ranges (the library's stem_owner_ranges), the all-to-all
keyed on kernel id, and the exact combination of the two global KKT scalars.
Each rank runs the ORACLE on the rows it owns; the union of the ranks' leaves
and the combined T / Ssum must equal the single-process oracle plan -- the
decomposition the CUDA dist path implements (ROOT decisions are local to a
kernel group; the KKT numerator is one exact sum, R12)."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle as O
import paper_conf_micro_chungnkk25_b200 as sr
from parity_util import Z95

WORLD = 2


def _trace():
    rng = np.random.default_rng(21)
    n, K = 6000, 23
    kid = (rng.zipf(1.4, n) % K).astype(np.uint32)
    t = (rng.integers(1, 9, K)[kid] * 1000 * rng.lognormal(0, 0.15, n)).astype(np.uint32)
    return kid, t, K


def _worker(rank, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=WORLD)
    kid, t, K = _trace()
    n = len(kid)
    lo, hi = n * rank // WORLD, n * (rank + 1) // WORLD
    my_kid, my_t, my_row = kid[lo:hi], t[lo:hi], np.arange(lo, hi)
    # 1. global kernel histogram
    cnt = torch.from_numpy(np.bincount(my_kid, minlength=K).astype(np.int64))
    dist.all_reduce(cnt)
    bounds = sr.owner_ranges(cnt.numpy().astype(np.uint64), WORLD)
    # 2. all-to-all keyed on kernel id (stable: each sender keeps its row order)
    dest = np.searchsorted(bounds[1:WORLD], my_kid, side="right")
    send = [torch.from_numpy(np.stack([my_kid[dest == d], my_t[dest == d], my_row[dest == d]]).astype(np.int64))
            for d in range(WORLD)]
    all_send = [None] * WORLD   # gloo has no variable all-to-all: every rank keeps what is addressed to it
    dist.all_gather_object(all_send, [x.numpy() for x in send])
    got = np.concatenate([all_send[s][rank] for s in range(WORLD)], axis=1)
    r_kid, r_t, r_row = got[0].astype(np.uint32), got[1].astype(np.uint32), got[2]
    assert np.all(np.diff(r_row) > 0)                       # arrives in global row order
    assert np.all((r_kid >= bounds[rank]) & (r_kid < bounds[rank + 1]))
    # 3. local ROOT leaves of the owned kernels (oracle), exact partial sums
    p = O.plan(r_kid, r_t, K, eps=0.05, z=Z95) if len(r_kid) else None
    leaves = np.zeros((0, 5), np.int64) if p is None else np.stack(
        [p["kernel_id"], p["ordinal"], p["lo_ns"], p["hi_ns"], p["n"]], 1).astype(np.int64)
    T = torch.tensor([0 if p is None else int(p["true_total_ns"])], dtype=torch.int64)
    dist.all_reduce(T)
    terms = [] if p is None else list(np.sqrt(p["mean_ns"] * (p["std_ns"] * p["n"]) ** 2))
    all_leaves = [None] * WORLD
    all_terms = [None] * WORLD
    dist.all_gather_object(all_leaves, leaves)
    dist.all_gather_object(all_terms, terms)
    if rank == 0:
        q.put((np.concatenate(all_leaves), int(T.item()), [x for tt in all_terms for x in tt]))
    dist.destroy_process_group()


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def test_owner_ranges_properties():
    rng = np.random.default_rng(4)
    for _ in range(200):
        K = int(rng.integers(1, 300))
        world = int(rng.integers(1, 9))
        c = rng.integers(0, 1000, K).astype(np.uint64) * (rng.random(K) < 0.8)
        b = sr.owner_ranges(c, world)
        assert b[0] == 0 and b[-1] == K and np.all(np.diff(b.astype(np.int64)) >= 0)
        tot, cum = int(c.sum()), np.concatenate([[0], np.cumsum(c.astype(np.int64))])
        for r in range(1, world):   # smallest k with cum[k] * world >= r * total
            k = int(b[r])
            assert cum[k] * world >= r * tot
            assert k == 0 or cum[k - 1] * world < r * tot or k == K


def test_gloo_world2_decomposition_matches_single_process():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, port, q)) for r in range(WORLD)]
    for p in procs:
        p.start()
    leaves, T, terms = q.get(timeout=240)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    kid, t, K = _trace()
    ref = O.plan(kid, t, K, eps=0.05, z=Z95)
    want = np.stack([ref["kernel_id"], ref["ordinal"], ref["lo_ns"], ref["hi_ns"], ref["n"]], 1).astype(np.int64)
    assert np.array_equal(leaves, want)                      # union of owned leaves == global leaves
    assert T == ref["true_total_ns"]                          # exact integer reduction
    assert O.exact_sum(np.array(terms)) == pytest.approx(ref["ssum"], rel=1e-12)
