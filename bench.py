#!/usr/bin/env python
"""Benchmark: trace rows/s to a STEM+ROOT sampling plan on B200 (BASELINE.json metric).

One step = one full pass of the hot path (a1 group/sort, a2 prefix moments,
a3/a4 ROOT levels, a5 leaf table, a6 STEM sizes, a7 Philox samples, a8
estimate + bound) over one synthetic trace already resident in HBM, through
the C ABI (stem_root_plan_ctx, plan left on the device).  Default workload:
BASELINE config C5 (1e9 invocations, 10k kernel ids), the configuration the
metric's 1/2/4/8-GPU figures are quoted on; it fits one B200.

    python bench.py [--gpus N --steps K --warmup W] [--config C5 --n ROWS] [--impl reference]

Prints ONE JSON line on rank 0.  See DESIGN.md §7 for every field.
"""
import argparse
import json
import os
import statistics
import subprocess
import sys
import tempfile
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "trace rows/sec to sampling plan"
UNIT = "rows/s"
WORKLOADS = {
    "C1": "C1 tiny: 10k invocations, 20 kernel ids, bimodal Gaussian, eps 5%, 95% conf",
    "C2": "C2 CASIO-shaped: 1M invocations, 500 kernel ids, unimodal/multimodal/gamma/lognormal mix",
    "C3": "C3 LLM-inference-shaped: 20M invocations, 2k kernel ids, lognormal + multi-saturation, 12 metrics",
    "C4": "C4 training-shaped: 100M invocations, 1k kernel ids, eps 5% (sweep 1-10% in tests)",
    "C5": "C5: 1e9 invocations, 10k kernel ids, LLM mix, Zipf(1.1) call sites",
}


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", choices=["ours", "reference"], default="ours")
    ap.add_argument("--config", default="C5")
    ap.add_argument("--n", type=int, default=None, help="override rows")
    ap.add_argument("--eps", type=float, default=None)
    ap.add_argument("--conf", type=float, default=0.95)
    ap.add_argument("--cpu-sample-rows", type=int, default=30_000_000)
    ap.add_argument("--ref-sample-rows", type=int, default=30_000_000)   # the same sample as cpu_baseline
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--split", type=int, default=0, choices=[0, 1, 2, 3], help="ROOT split rule: 0 exact 2-means (default), 1 Lloyd (R26), 2 k-means++ seeded Lloyd (R27), 3 exact k-means with --kmeans-k groups (R29)")
    ap.add_argument("--kmeans-k", type=int, default=3, help="groups per ROOT split with --split 3 (2..8)")
    ap.add_argument("--metric-bounds", action="store_true", help="also true totals and bounds of the metric columns (R28)")
    ap.add_argument("--dry-launch", action="store_true", help="print the torchrun command --gpus N would run, and exit")
    return ap.parse_args()


def launch(a):
    """--gpus N without a torchrun environment: re-exec this script under torchrun
    with N ranks (one per GPU, rendezvous on 127.0.0.1).  Under torchrun the rank
    count must equal --gpus.  Our arm needs N visible CUDA devices and fails
    loudly otherwise (never a silent 1-GPU run)."""
    ws = os.environ.get("WORLD_SIZE")
    if ws is not None:
        if int(ws) != a.gpus:
            print(json.dumps({"metric": METRIC, "error": f"WORLD_SIZE={ws} but --gpus {a.gpus}"}), flush=True)
            sys.exit(2)
        return
    if a.gpus <= 1:
        return
    if a.impl == "ours" and not a.dry_launch:
        import torch
        have = torch.cuda.device_count()
        if have < a.gpus:
            print(json.dumps({"metric": METRIC, "error": f"--gpus {a.gpus} requested but {have} CUDA devices are "
                              "visible"}), flush=True)
            sys.exit(2)
    import socket
    with socket.socket() as so:
        so.bind(("127.0.0.1", 0))
        port = so.getsockname()[1]
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={a.gpus}",
           "--master-addr=127.0.0.1", f"--master-port={port}", os.path.abspath(__file__)] + \
        [x for x in sys.argv[1:] if x != "--dry-launch"]
    if a.dry_launch:
        print(json.dumps({"launch": cmd}), flush=True)
        sys.exit(0)
    sys.exit(subprocess.call(cmd))


def load_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, copy kernel)"
    return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


def load_ncu_traffic():
    """Per-launch DRAM bytes of our kernels from the committed ncu --set full summary."""
    p = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if os.path.exists(p):
        with open(p) as f:
            return json.load(f)
    return {}


class Clocks:
    """nvidia-smi sampling during the timed region (B200_PROFILING.md clocks line)."""
    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, dev):
        self.dev = dev
        self.f = tempfile.NamedTemporaryFile("w+", suffix=".csv", delete=False)
        self.p = None

    def start(self):
        try:
            self.p = subprocess.Popen(["nvidia-smi", f"--id={self.dev}", f"--query-gpu={self.Q}",
                                       "--format=csv,noheader,nounits", "-lms", "100"], stdout=self.f,
                                      stderr=subprocess.DEVNULL)
        except OSError:
            self.p = None

    def stop(self):
        if self.p is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.p.terminate()
        self.p.wait()
        self.f.flush()
        rows = []
        with open(self.f.name) as f:
            for line in f:
                parts = [x.strip() for x in line.split(",")]
                if len(parts) >= 9:
                    rows.append(parts)
        os.unlink(self.f.name)
        if not rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["no samples"]}
        sm = [float(r[1]) for r in rows if r[1].replace(".", "").isdigit()]
        mx = [float(r[2]) for r in rows if r[2].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for r in rows for i in range(4) if r[5 + i].lower() == "active"})
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(rows)}


def dist_env():
    return int(os.environ.get("RANK", 0)), int(os.environ.get("WORLD_SIZE", 1)), int(os.environ.get("LOCAL_RANK", 0))


SPLIT_NAMES = ["exact optimal 2-means (R5)", "Lloyd k-means, k = 2 (R26)", "k-means++ seeded Lloyd, k = 2 (R27)",
               "exact optimal k-means, k = {k} (R29)"]


def split_name(a):
    return SPLIT_NAMES[a.split].format(k=a.kmeans_k)


def run_reference(a):
    """--impl reference: the oracle (plain single-threaded C, oracle/) as it stands, on the
    host cores, on a bounded sample of the same workload; rank 0 only."""
    rank, world, _ = dist_env()
    if rank != 0:
        return
    import numpy as np

    import oracle
    import tracegen
    sp = tracegen.spec(a.config, n=a.n)
    m = min(a.ref_sample_rows, sp.n)
    kid, t, met = tracegen.generate_np(sp, 0, m)
    eps = a.eps if a.eps is not None else sp.eps
    z = 1.959963984540054
    times = []
    for i in range(a.warmup + a.steps):
        t0 = time.perf_counter()
        oracle.plan(kid, t, sp.n_kernels, eps=eps, z=z, seed=i, metrics=met, split=a.split,
                    metric_bounds=int(a.metric_bounds), kmeans_k=a.kmeans_k)
        dt = time.perf_counter() - t0
        if i >= a.warmup:
            times.append(dt)
    tot = sum(times)
    value = m * len(times) / tot
    line = {
        "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": a.steps, "warmup": a.warmup,
        "ms_per_step": 1e3 * tot / len(times), "higher_is_better": True, "scaling": "strong", "vs_baseline": None,
        "dtype": "u32 keys, exact int64/int128 moments, f64", "data": "synthetic (tracegen, seeded)",
        "impl": "reference",
        "config": {"workload": WORKLOADS.get(a.config, a.config), "rows": sp.n, "kernels": sp.n_kernels,
                   "eps": eps, "conf": a.conf, "split": split_name(a), "sample_rows": m},
        "cpu_baseline": {"value": value, "unit": UNIT, "cores": 1, "kind": "oracle",
                         "sample": f"first {m} rows of {a.config} (oracle single-threaded C, -O2)"},
        "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
        "gpu_launches": 0,
    }
    print(json.dumps(line), flush=True)


def run_ours(a):
    import numpy as np
    import torch

    import paper_conf_micro_chungnkk25_b200 as sr
    import tracegen

    rank, world, local = dist_env()
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        import torch.distributed as dist
        dist.init_process_group("nccl", device_id=dev)
    sp = tracegen.spec(a.config, n=a.n)
    eps = a.eps if a.eps is not None else sp.eps
    # rows of this rank: the whole trace at N=1; at N>1 the contiguous row shard
    # [r N/W, (r+1) N/W) of the same global trace (strong scaling); stem_root_plan_dist
    # exchanges rows by kernel id over NCCL and gathers the plan on rank 0
    row0 = sp.n * rank // world
    n_local = sp.n * (rank + 1) // world - row0
    comm = None
    if world > 1:
        uid = torch.zeros(128, dtype=torch.uint8, device=dev)
        if rank == 0:
            uid.copy_(torch.frombuffer(bytearray(sr.nccl_unique_id()), dtype=torch.uint8))
        torch.distributed.broadcast(uid, 0)
        comm = sr.Comm.nccl(bytes(uid.cpu().numpy()), rank, world, local)
    ds = tracegen.DeviceSpec(sp, dev)
    kid = torch.empty(n_local, dtype=torch.int32, device=dev)
    tt = torch.empty(n_local, dtype=torch.int32, device=dev)
    nm = sp.n_metrics
    met = torch.empty((nm, n_local), dtype=torch.float64, device=dev) if nm else None
    tracegen.generate_cuda(ds, kid, tt, met, row0=row0, count=n_local)
    torch.cuda.synchronize()
    del ds

    ctx = sr.Context(local)
    stream = torch.cuda.current_stream(dev)

    def step():
        # one whole plan through the C ABI, ending with the plan in host memory
        # (rows/s up to "the plan on host"); rank 0 gets the plan
        hp = ctx.plan_host_raw(kid, tt, sp.n_kernels, eps=eps, conf=a.conf, metrics=met, comm=comm,
                               global_row_base=row0, seed=12345, stream=stream.cuda_stream, split=a.split,
                               metric_bounds=a.metric_bounds, kmeans_k=a.kmeans_k)
        nb = hp.nbytes()
        hp.close()
        return nb

    for _ in range(a.warmup):
        step()
    torch.cuda.synchronize()
    # timed region (device time, CUDA events on the plan's stream; per-stage events live)
    ctx.enable_timing(True)
    stages = {}
    clocks = Clocks(local)
    clocks.start()
    if world > 1:
        torch.distributed.barrier()
    torch.cuda.synchronize()
    ev0 = torch.cuda.Event(enable_timing=True)
    ev1 = torch.cuda.Event(enable_timing=True)
    ev0.record(stream)
    launches = 0
    plan_bytes = 0
    for _ in range(a.steps):
        plan_bytes = step()
        for s in ctx.stage_times():
            g = stages.setdefault(s["name"], {"ms": 0.0, "bytes": 0, "launches": 0, "count": 0})
            for k in ("ms", "bytes", "launches", "count"):
                g[k] += s[k]
        launches += ctx.stats()["kernel_launches"]
    ev1.record(stream)
    torch.cuda.synchronize()
    if world > 1:
        torch.distributed.barrier()
    ck = clocks.stop()
    ctx.enable_timing(False)
    elapsed_ms = ev0.elapsed_time(ev1)
    if world > 1:
        tmax = torch.tensor([elapsed_ms], device=dev)
        torch.distributed.all_reduce(tmax, op=torch.distributed.ReduceOp.MAX)
        elapsed_ms = float(tmax.item())
    st = ctx.stats()
    dplan = ctx.device_plan()
    ms_per_step = elapsed_ms / a.steps
    # rows each rank grouped and clustered after the kernel-id exchange (SURVEY §8(e) skew caveat)
    owned = [int(st["owned_rows"])]
    if world > 1:
        owned = [None] * world
        torch.distributed.all_gather_object(owned, int(st["owned_rows"]))
    balance = {"rows_per_rank": owned, "max_over_mean": max(owned) / (sum(owned) / len(owned)) if sum(owned) else 1.0,
               "comm_ranks": int(st["world"])}
    value = sp.n * a.steps / (elapsed_ms / 1e3)

    # roofline of the dominant kernel (largest share of the step)
    peak, peak_src = load_peaks()
    dom = max(stages.items(), key=lambda kv: kv[1]["ms"])
    per_launch_bytes = dom[1]["bytes"] / max(dom[1]["count"], 1)
    per_launch_ms = dom[1]["ms"] / max(dom[1]["count"], 1)
    achieved = per_launch_bytes / (per_launch_ms * 1e-3) / 1e9
    traffic = load_ncu_traffic().get(a.config, {}).get(dom[0])
    roofline = {"bound": "hbm", "kernel": dom[0], "achieved": achieved, "peak": peak, "unit": "GB/s",
                "frac": achieved / peak, "traffic": traffic, "peak_source": peak_src,
                "algorithmic_bytes_per_launch": per_launch_bytes, "ms_per_launch": per_launch_ms,
                "share_of_step": dom[1]["ms"] / a.steps / ms_per_step}
    all_bytes = sum(v["bytes"] for v in stages.values()) / a.steps
    path = {"algorithmic_bytes_per_step": all_bytes,
            "achieved_gbs_over_step": all_bytes / (ms_per_step * 1e-3) / 1e9}

    line = {
        "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": a.steps, "warmup": a.warmup,
        "ms_per_step": ms_per_step, "higher_is_better": True, "scaling": "strong", "vs_baseline": None,
        "dtype": "u32 keys, exact int64/int128 moments, f64", "data": "synthetic (tracegen, seeded, on device)",
        "config": {"workload": WORKLOADS.get(a.config, a.config), "rows": sp.n,
                   "kernels": sp.n_kernels, "eps": eps, "conf": a.conf, "metrics": nm,
                   "split": split_name(a),
                   "parallelism": "single GPU" if world == 1 else
                   f"{world} GPUs: row shards, NCCL all-to-all by kernel id, exact allreduce",
                   "l2": "inputs 8 B/row x rows >> 126 MB L2 (no flush needed)" if n_local >= 50_000_000
                   else "inputs fit in L2: latency-bound workload",
                   "sort_key_bits": st["key_bits"], "sort_passes": st["sort_passes"],
                   "sort_row_bits_in_key": st["pack_bits"], "ambiguous_samples": st["ambiguous_samples"],
                   "split_chunks": st["split_chunks"], "split_scanned": st["split_scanned"],
                   "root_levels": st["levels"], "clusters": st["n_clusters"], "samples": st["n_samples"],
                   "active_rows_over_levels": st["active_rows"], "plan_to_host": True,
                   "plan_bytes_d2h": plan_bytes, "metric_bounds": bool(a.metric_bounds)},
        "balance": balance,
        "clocks": ck,
        "gpu_launches": launches,
        "roofline": roofline,
        "path": path,
        "stages_ms_per_step": {k: v["ms"] / a.steps for k, v in sorted(stages.items(), key=lambda kv: -kv[1]["ms"])},
    }

    # e2e: same metric through the public API with HOST buffers (pinned), host plan out
    if not a.no_e2e:
        hk = torch.empty(n_local, dtype=torch.int32, pin_memory=True)
        ht = torch.empty(n_local, dtype=torch.int32, pin_memory=True)
        hk.copy_(kid)
        ht.copy_(tt)
        hm = None
        if nm:
            hm = torch.empty((nm, n_local), dtype=torch.float64, pin_memory=True)
            hm.copy_(met)
        torch.cuda.synchronize()
        e2e_steps = max(1, min(a.steps, 3))
        d2h = 0
        def e2e_step():
            # the C-ABI call with HOST buffers: the library copies the trace in and returns the
            # host plan (stem_plan); the plan's bytes are what crosses back
            hp = ctx.plan_host_raw(hk, ht, sp.n_kernels, eps=eps, conf=a.conf, metrics=hm, comm=comm,
                                   global_row_base=row0, seed=12345, stream=stream.cuda_stream, split=a.split,
                                   metric_bounds=a.metric_bounds, kmeans_k=a.kmeans_k)
            nb = hp.nbytes()
            hp.close()
            return nb
        d2h = e2e_step()
        torch.cuda.synchronize()
        if world > 1:
            torch.distributed.barrier()
        t0 = time.perf_counter()
        for _ in range(e2e_steps):
            d2h = e2e_step()
        e2e_s = (time.perf_counter() - t0) / e2e_steps
        if world > 1:
            tm = torch.tensor([e2e_s], device=dev, dtype=torch.float64)
            torch.distributed.all_reduce(tm, op=torch.distributed.ReduceOp.MAX)
            e2e_s = float(tm.item())
        line["e2e"] = {"value": sp.n / e2e_s, "unit": UNIT,
                       "h2d_bytes_per_step": sp.n * (8 + 8 * nm), "d2h_bytes_per_step": int(d2h),
                       "ms_per_step": e2e_s * 1e3, "steps": e2e_steps}
        del hk, ht, hm

    # cpu_baseline: the oracle as it stands, on a bounded sample of the same workload (rank 0, N=1)
    if not a.no_cpu_baseline and rank == 0 and world == 1:
        import oracle
        m = min(a.cpu_sample_rows, n_local)
        k_np = kid[:m].cpu().numpy().view(np.uint32)
        t_np = tt[:m].cpu().numpy().view(np.uint32)
        m_np = met[:, :m].cpu().numpy() if nm else None
        t0 = time.perf_counter()
        oracle.plan(k_np, t_np, sp.n_kernels, eps=eps, z=dplan["z"], seed=12345, metrics=m_np, split=a.split,
                    metric_bounds=int(a.metric_bounds), kmeans_k=a.kmeans_k)
        cs = time.perf_counter() - t0
        line["cpu_baseline"] = {"value": m / cs, "unit": UNIT, "cores": 1, "kind": "oracle",
                                "sample": f"first {m} rows of {a.config} ({cs:.1f} s, single-threaded C oracle)",
                                "host_nproc": os.cpu_count()}
    if rank == 0:
        print(json.dumps(line), flush=True)
    ctx.close()
    if comm is not None:
        comm.close()
    if world > 1:
        torch.distributed.destroy_process_group()


def main():
    a = parse()
    launch(a)
    if a.impl == "reference":
        run_reference(a)
    else:
        run_ours(a)


if __name__ == "__main__":
    main()
