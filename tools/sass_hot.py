"""Top SASS instructions of an ncu report by warp-stall samples, with their stall reasons.

    python tools/sass_hot.py report.ncu-rep [N] [kernel-regex]"""
import csv
import io
import subprocess
import sys


def main():
    rep, top = sys.argv[1], int(sys.argv[2]) if len(sys.argv) > 2 else 30
    filt = ["-k", "regex:" + sys.argv[3]] if len(sys.argv) > 3 else []
    out = subprocess.check_output(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"] + filt,
                                  stderr=subprocess.DEVNULL).decode()
    r = list(csv.reader(io.StringIO(out)))
    h = r[1]
    rows = []
    for x in r[2:]:   # the first kernel's section only
        if x and x[0].startswith("Kernel Name"):
            break
        if len(x) == len(h):
            rows.append(x)
    ix = {k: i for i, k in enumerate(h)}
    S = ix["Warp Stall Sampling (All Samples)"]
    E = ix["Instructions Executed"]
    tot = sum(float(x[S] or 0) for x in rows) or 1.0
    cols = [c for c in h if c.startswith("stall_") and "Not Issued" not in c]
    print(f"{r[0][0][:100]}: {len(rows)} instructions, {tot:.0f} samples, "
          f"{sum(float(x[E] or 0) for x in rows):.3g} warp instructions executed")
    for s, i, x in sorted(((float(x[S] or 0), i, x) for i, x in enumerate(rows)), reverse=True)[:top]:
        det = " ".join(f"{c[6:]}={x[ix[c]]}" for c in cols if x[ix[c]] not in ("0", ""))
        print(f"{i:5d} {s / tot * 100:5.1f}% {x[ix['Source']][:64]:64s} {det}")


if __name__ == "__main__":
    main()
