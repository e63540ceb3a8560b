"""Sort-stage (a1) microbenchmark: builds the library sources + sb.cu into
tools/sortbench/build/libsb_<tag>.so for each compile-time variant (-D...), runs
sort_trace on a device-resident tracegen trace, prints per-stage ms and checks
the output against torch's stable sort (--check).

  python tools/sortbench/sortbench.py [--config C5] [--n N] [--check] "" "-DSR_X=1" ...
"""
import argparse
import ctypes as C
import hashlib
import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(os.path.dirname(HERE))
sys.path.insert(0, ROOT)


def build(defs):
    import paper_conf_micro_chungnkk25_b200 as m
    tag = hashlib.md5(defs.encode()).hexdigest()[:8]
    out = os.path.join(HERE, "build", f"libsb_{tag}.so")
    srcs = [os.path.join(m._CSRC, s) for s in m.SOURCES] + [os.path.join(HERE, "sb.cu")]
    if not os.path.exists(out) or os.path.getmtime(out) < max(map(os.path.getmtime, srcs + [os.path.join(m._CSRC, "internal.h")])):
        os.makedirs(os.path.dirname(out), exist_ok=True)
        cmd = ["nvcc"] + m.NVCC_FLAGS + defs.split() + ["-I", m._nccl_include(), "-o", out] + srcs + ["-ldl"]
        subprocess.check_call(cmd, cwd=m._CSRC)
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C5")
    ap.add_argument("--n", type=int, default=None)
    ap.add_argument("--warm", type=int, default=2)
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--check", action="store_true")
    ap.add_argument("--build-only", action="store_true")
    ap.add_argument("variants", nargs="*", default=[""])
    a = ap.parse_args()
    libs = [(v, build(v)) for v in a.variants]
    if a.build_only:
        return
    import torch
    import tracegen as G
    sp = G.spec(a.config, n=a.n)
    n = sp.n
    kid = torch.empty(n, dtype=torch.int32, device="cuda")
    t = torch.empty(n, dtype=torch.int32, device="cuda")
    G.generate_cuda(G.DeviceSpec(sp, "cuda"), kid, t)
    torch.cuda.synchronize()
    ref = None
    for v, path in libs:
        lib = C.CDLL(path)
        ms = (C.c_double * 32)()
        names = C.create_string_buffer(32 * 32)
        pb = C.c_int(0)
        tc = torch.empty(n, dtype=torch.int32, device="cuda") if a.check else None
        rc_ = torch.empty(n, dtype=torch.int32, device="cuda") if a.check else None
        rc = lib.sb_sort(C.c_void_p(kid.data_ptr()), C.c_void_p(t.data_ptr()), C.c_uint64(n), C.c_uint32(sp.n_kernels),
                         a.warm, a.reps, ms, names, 32, C.c_void_p(tc.data_ptr() if a.check else 0),
                         C.c_void_p(rc_.data_ptr() if a.check else 0), C.byref(pb))
        if rc > -1000:
            print(f"[{v}] FAILED rc={rc}")
            continue
        nst = -1000 - rc
        st = {names.raw[32 * j:32 * j + 32].split(b"\0")[0].decode(): ms[j] for j in range(nst)}
        tot = sum(st.values())
        line = " ".join(f"{k}={x:.3f}" for k, x in st.items())
        ok = ""
        if a.check:
            if ref is None:
                key = (kid.to(torch.int64) << 32) | (t.to(torch.int64) & 0xFFFFFFFF)
                _, idx = torch.sort(key, stable=True)
                del key
                ref = (t[idx], idx)
            mask = (1 << pb.value) - 1 if pb.value else 0xFFFFFFFF
            ok_t = bool(torch.equal(tc, ref[0]))
            ok_r = bool(torch.equal(rc_.to(torch.int64) & 0xFFFFFFFF & mask, ref[1] & mask))
            ok = f" check t={'OK' if ok_t else 'BAD'} row={'OK' if ok_r else 'BAD'}"
        print(f"[{v}] total {tot:.3f} ms | {line}{ok}", flush=True)
        del tc, rc_


if __name__ == "__main__":
    main()
