"""One small run of every path of the library, for compute-sanitizer
(tests/test_gpu_sanitizer.py):  python tools/sanitize_run.py C1|C2 [quick]

Covers the sort passes (decoupled look-back spin on published statuses), the
pipelined ROOT level loop (frontier sizes read from HBM by the next level),
the three split rules, the leaf table / STEM sizes / sampler / estimator,
metric_bounds, the host-pointer path and a 2-rank loopback plan."""
import os
import sys
import threading

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_micro_chungnkk25_b200 as sr  # noqa: E402
import tracegen as G  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "C1"
quick = len(sys.argv) > 2 and sys.argv[2] == "quick"
sp = G.spec(name, n=min(G.spec(name).n, 200_000))
kid, t, _ = G.generate_np(sp)
met = np.vstack([t.astype(np.float64), np.random.default_rng(1).random(len(t))])
dk = torch.from_numpy(kid.view(np.int32)).cuda()
dt = torch.from_numpy(t.view(np.int32)).cuda()
dm = torch.from_numpy(met).cuda()
ctx = sr.Context(0)
z = 1.959963984540054
ctx.plan(dk, dt, sp.n_kernels, eps=0.02, z=z, seed=1, metrics=dm, metric_bounds=True)
if not quick:
    for split in (1, 2):
        ctx.plan(dk, dt, sp.n_kernels, eps=0.02, z=z, seed=2, split=split)
    ctx.plan(kid, t, sp.n_kernels, eps=0.05, z=z, seed=3, metrics=met, scope=1, census_cap=True)
    comms = sr.Comm.loopback(2, 0)
    ctxs = [sr.Context(0) for _ in range(2)]
    cut = len(kid) // 2
    shards = [(dk[:cut], dt[:cut], dm[:, :cut].contiguous()), (dk[cut:], dt[cut:], dm[:, cut:].contiguous())]
    streams = [torch.cuda.Stream() for _ in range(2)]
    err = []

    def run(r):
        try:
            k, tt, m = shards[r]
            ctxs[r].plan_dist(comms[r], k, tt, sp.n_kernels, r * cut, eps=0.02, z=z, seed=4, metrics=m,
                              metric_bounds=True, stream=streams[r].cuda_stream)
        except Exception as e:  # noqa: BLE001
            err.append(e)
    th = [threading.Thread(target=run, args=(r,)) for r in range(2)]
    for x in th:
        x.start()
    for x in th:
        x.join()
    if err:
        raise err[0]
torch.cuda.synchronize()
print("SANITIZE_RUN_OK", flush=True)
