"""Sampling-quality harness: how good are the plans the
library builds, measured the way the paper measures its methods, on the seeded
synthetic traces of tracegen (no paper data is needed or used).

For each method and each of R sampling seeds on one trace:
  * sampling error  e = |t_total - t*| / t* x 100 %            (Eq. 1)
  * speedup         t* / (sum of t over the distinct sampled invocations)
                    ("cycle count of the full workload to that of the sampled
                    workload"; a duplicate draw is simulated once)
  * the predicted bound eps_pred of the plan (Eq. 5) and whether e <= it.
Aggregates follow P:L258: arithmetic mean of the error, harmonic mean of the
speedup over the seeds.

Methods:
  stem+root   the library's default plan (ROOT on, global joint Eq. 6)
  stem        ROOT off: one cluster per kernel (Eq. 6 over kernel groups)
  per-kernel  ROOT on, Eq. 6 solved per kernel (scope 1, union bound Thm. 3.1)
  per-leaf    ROOT on, Eq. 3 per leaf (scope 2)
  lloyd       ROOT with Lloyd's k-means (k = 2) instead of the exact 2-means cut
              (opts.split = 1, R26: the paper's "k-means")
  kmeans++    the same from k-means++ seeds (opts.split = 2, R27; the tree changes
              with every sampling seed, like a randomly seeded library k-means)
  kmeans-3/4  ROOT splitting each cluster into 3 / 4 groups by the exact k-means
              (opts.split = 3, R29: "any number above 2 works well")
  random-p    uniform random sampling, each invocation kept with probability p,
              estimate sum(t)/p (the paper's baseline)
and an eps sweep of stem+root (Fig. 11).  Configs with metric columns
(C3) add the metric estimates: per column the relative error of the
weighted sum against the exact total, and how often it lies inside the
predicted metric bound (metric_bounds, R28).

    python tools/quality.py [--config C2] [--n ROWS] [--seeds 20] [--eps 0.03,0.05,0.1,0.25]
                            [--out profiles/r01_quality_C2.json]

Needs a GPU (the plans come from libstemroot.so through the Python binding)."""
import argparse
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def _hmean(x):
    x = np.asarray(x, dtype=np.float64)
    return float(len(x) / np.sum(1.0 / x))


def _summary(err, spd, bound=None, eps=None, samples=None):
    out = {"mean_error_pct": float(np.mean(err)), "max_error_pct": float(np.max(err)),
           "hmean_speedup": _hmean(spd), "runs": len(err)}
    if bound is not None:
        out["mean_bound_pct"] = float(np.mean(bound))
        out["coverage_of_bound"] = float(np.mean(np.asarray(err) <= np.asarray(bound)))
    if eps is not None:
        out["coverage_of_eps"] = float(np.mean(np.asarray(err) <= 100.0 * eps))
    if samples is not None:
        out["mean_samples"] = float(np.mean(samples))
    return out


def plan_quality(ctx, kid, t, n_kernels, t64, total, eps, seeds, **opts):
    """Error / speedup / bound of the library's plan over sampling seeds.
    kid, t: device tensors (int32 views); t64: the same times as int64 (device)."""
    import torch
    err, spd, bnd, ns = [], [], [], []
    for s in seeds:
        p = ctx.plan(kid, t, n_kernels, eps=eps, seed=int(s), **opts)
        assert p["true_total_ns"] == total
        err.append(100.0 * abs(p["est_total_ns"] - total) / total)
        rows = torch.from_numpy(np.unique(p["sample_row"]).astype(np.int64)).to(t64.device)
        spd.append(total / float(t64[rows].sum().item()))
        bnd.append(100.0 * p["bound"])
        ns.append(len(p["sample_row"]))
    return _summary(err, spd, bnd, eps, ns)


def metric_quality(ctx, kid, t, sp, eps, seeds, kw):
    """Per metric column: mean / max relative error of the weighted-sum estimate
     against the exact total, the mean predicted bound and its coverage."""
    import torch
    import tracegen as G
    _, _, met_np = G.generate_np(sp)
    met = torch.from_numpy(met_np).cuda()
    errs, bnds = [], []
    for s in seeds:
        p = ctx.plan(kid, t, sp.n_kernels, eps=eps, seed=int(s), metrics=met, metric_bounds=True, **kw)
        tru = np.asarray(p["true_metric"])
        errs.append(100.0 * np.abs(np.asarray(p["est_metric"]) - tru) / np.abs(tru))
        bnds.append(100.0 * np.asarray(p["bound_metric"]))
    e, b = np.array(errs), np.array(bnds)
    return {"columns": int(e.shape[1]), "mean_error_pct": e.mean(axis=0).tolist(),
            "max_error_pct": e.max(axis=0).tolist(), "mean_bound_pct": b.mean(axis=0).tolist(),
            "coverage_of_bound": (e <= b).mean(axis=0).tolist(), "coverage_all": float((e <= b).mean())}


def random_quality(t64, total, prob, seeds):
    """Uniform random sampling baseline: Bernoulli(prob) per invocation,
    Horvitz-Thompson estimate sum(t) / prob."""
    import torch
    err, spd = [], []
    for s in seeds:
        g = torch.Generator(device=t64.device)
        g.manual_seed(int(s))
        keep = torch.rand(t64.shape[0], generator=g, device=t64.device) < prob
        st = float(t64[keep].sum().item())
        err.append(100.0 * abs(st / prob - total) / total)
        spd.append(total / max(st, 1.0))
    return _summary(err, spd)


def run(config="C2", n=None, n_seeds=20, eps_list=(0.03, 0.05, 0.1, 0.25), z=0.0):
    import torch

    import paper_conf_micro_chungnkk25_b200 as sr
    import tracegen as G

    sp = G.spec(config, n=n)
    if sp.n > 50_000_000 and not sp.n_metrics:   # bench-size traces: the byte-identical CUDA twin
        kid = torch.empty(sp.n, dtype=torch.int32, device="cuda")
        t = torch.empty(sp.n, dtype=torch.int32, device="cuda")
        G.generate_cuda(G.DeviceSpec(sp, "cuda"), kid, t)
    else:
        kid_np, t_np, _ = G.generate_np(sp)
        kid = torch.from_numpy(kid_np.view(np.int32)).cuda()
        t = torch.from_numpy(t_np.view(np.int32)).cuda()
    t64 = t.to(torch.int64) & 0xFFFFFFFF
    total = int(t64.sum().item())
    seeds = [1000 + i for i in range(n_seeds)]
    ctx = sr.Context(0)
    eps = sp.eps
    res = {"config": config, "rows": sp.n, "kernels": sp.n_kernels, "eps": eps, "seeds": n_seeds,
           "z": z if z > 0 else "Phi^-1(1 - alpha/2), conf 0.95", "methods": {}, "eps_sweep": {}}
    kw = dict(z=z)
    res["methods"]["stem+root"] = plan_quality(ctx, kid, t, sp.n_kernels, t64, total, eps, seeds, **kw)
    res["methods"]["stem"] = plan_quality(ctx, kid, t, sp.n_kernels, t64, total, eps, seeds, root=False, **kw)
    res["methods"]["per-kernel"] = plan_quality(ctx, kid, t, sp.n_kernels, t64, total, eps, seeds, scope=1, **kw)
    res["methods"]["per-leaf"] = plan_quality(ctx, kid, t, sp.n_kernels, t64, total, eps, seeds, scope=2, **kw)
    res["methods"]["lloyd"] = plan_quality(ctx, kid, t, sp.n_kernels, t64, total, eps, seeds, split=1, **kw)
    res["methods"]["kmeans++"] = plan_quality(ctx, kid, t, sp.n_kernels, t64, total, eps, seeds, split=2, **kw)
    for k in (3, 4):
        res["methods"][f"kmeans-{k}"] = plan_quality(ctx, kid, t, sp.n_kernels, t64, total, eps, seeds, split=3,
                                                     kmeans_k=k, **kw)
    if sp.n_metrics:
        res["metrics"] = metric_quality(ctx, kid, t, sp, eps, seeds, kw)
    for prob in (0.001, 0.1):
        res["methods"][f"random-{prob:g}"] = random_quality(t64, total, prob, seeds)
    for e in eps_list:
        res["eps_sweep"][f"{e:g}"] = plan_quality(ctx, kid, t, sp.n_kernels, t64, total, e, seeds, **kw)
    ctx.close()
    return res


def _print(res):
    print(f"{res['config']}: {res['rows']} rows, {res['kernels']} kernels, eps {res['eps']}, {res['seeds']} seeds")
    if "metrics" in res:
        m = res["metrics"]
        print(f"metrics: {m['columns']} columns, mean error % " + " ".join(f"{x:.3f}" for x in m["mean_error_pct"]) +
              f"; mean bound % " + " ".join(f"{x:.3f}" for x in m["mean_bound_pct"]) +
              f"; coverage {m['coverage_all']:.2f}")
    print(f"{'method':<14} {'mean err %':>10} {'max err %':>10} {'hmean speedup':>14} {'bound %':>8} "
          f"{'cov(bound)':>10} {'samples':>9}")
    rows = list(res["methods"].items()) + [(f"eps={k}", v) for k, v in res["eps_sweep"].items()]
    for k, v in rows:
        print(f"{k:<14} {v['mean_error_pct']:10.4f} {v['max_error_pct']:10.4f} {v['hmean_speedup']:14.1f} "
              f"{v.get('mean_bound_pct', float('nan')):8.3f} {v.get('coverage_of_bound', float('nan')):10.2f} "
              f"{v.get('mean_samples', float('nan')):9.0f}")


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C2")
    ap.add_argument("--n", type=int, default=None)
    ap.add_argument("--seeds", type=int, default=20)
    ap.add_argument("--eps", default="0.03,0.05,0.1,0.25")
    ap.add_argument("--z", type=float, default=0.0)
    ap.add_argument("--out", default=None)
    a = ap.parse_args()
    res = run(a.config, a.n, a.seeds, tuple(float(x) for x in a.eps.split(",")), a.z)
    _print(res)
    if a.out:
        with open(a.out, "w") as f:
            json.dump(res, f, indent=1)


if __name__ == "__main__":
    main()
