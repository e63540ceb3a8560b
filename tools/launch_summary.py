"""Summarise an ncu launch list (gpu__time_duration.sum CSV) by kernel: count, total ms, share."""
import collections
import csv
import re
import sys


def summarise(path, skip_prefix=("gen_kernel",)):
    rows = [r for r in csv.reader(open(path)) if len(r) > 10]
    hdr = rows[0]
    ki, vi, ui = hdr.index("Kernel Name"), hdr.index("Metric Value"), hdr.index("Metric Unit")
    scale = {"ns": 1e-6, "nsecond": 1e-6, "us": 1e-3, "usecond": 1e-3, "ms": 1.0, "msecond": 1.0}
    agg = collections.OrderedDict()
    for r in rows[1:]:
        name = re.sub(r"^(void |<unnamed>::)", "", r[ki])
        name = re.sub(r"\(.*", "", name.replace("sr::", ""))
        if name.startswith(skip_prefix):
            continue
        v = float(r[vi].replace(",", "")) * scale[r[ui]]
        a = agg.setdefault(name, [0, 0.0])
        a[0] += 1
        a[1] += v
    return agg


if __name__ == "__main__":
    agg = summarise(sys.argv[1])
    tot = sum(v[1] for v in agg.values())
    print(f"{'ms':>10} {'share':>6} {'launches':>8}  kernel")
    for k, v in sorted(agg.items(), key=lambda kv: -kv[1][1]):
        print(f"{v[1]:10.3f} {100 * v[1] / tot:5.1f}% {v[0]:8d}  {k[:110]}")
    print(f"{tot:10.3f} total ms ({sum(v[0] for v in agg.values())} launches)")
