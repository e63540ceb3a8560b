"""Per-level device times of the ROOT split kernels from an ncu launch list
(the last step of the run):  python tools/level_table.py launches.csv"""
import csv
import re
import sys

rows = [r for r in csv.reader(open(sys.argv[1])) if len(r) > 10]
h = rows[0]
ki, vi, ui = h.index("Kernel Name"), h.index("Metric Value"), h.index("Metric Unit")
sc = {"ns": 1e-6, "nsecond": 1e-6, "us": 1e-3, "usecond": 1e-3, "ms": 1.0, "msecond": 1.0}
seq = [(re.sub(r"\(.*", "", r[ki].replace("sr::", "").replace("void ", "")).split("<")[0],
        float(r[vi].replace(",", "")) * sc[r[ui]]) for r in rows[1:]]
starts = [i for i, (k, _) in enumerate(seq) if k.startswith("prepass")]
step = seq[starts[-1]:]
levels, cur = [], {}
for k, v in step:
    if "entries" in k or k.startswith("nc_split"):
        if cur:
            levels.append(cur)
        cur = {}
    if any(x in k for x in ("big", "small", "decide", "lloyd", "nc_split")):
        cur[k] = cur.get(k, 0.0) + v
levels.append(cur)
tot = {}
for i, c in enumerate(levels):
    print(f"{i + 1:3d} " + " ".join(f"{k.replace('_kernel', '')}={v * 1000:.0f}us" for k, v in c.items()))
    for k, v in c.items():
        tot[k] = tot.get(k, 0.0) + v
print("total " + " ".join(f"{k.replace('_kernel', '')}={v:.3f}ms" for k, v in tot.items()))
