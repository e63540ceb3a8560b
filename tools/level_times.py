"""Per-level device times of the ROOT kernels from an ncu launch list (second step of the run).

    python tools/level_times.py launches.csv"""
import csv
import re
import sys

rows = [r for r in csv.reader(open(sys.argv[1])) if len(r) > 10]
h = rows[0]
ki, vi, ui = h.index("Kernel Name"), h.index("Metric Value"), h.index("Metric Unit")
sc = {"ns": 1e-6, "nsecond": 1e-6, "us": 1e-3, "usecond": 1e-3, "ms": 1.0, "msecond": 1.0}
seq = [(re.sub(r"\(.*", "", r[ki].replace("sr::", "").replace("void ", "")), float(r[vi].replace(",", "")) * sc[r[ui]])
       for r in rows[1:]]
starts = [i for i, (k, _) in enumerate(seq) if k.startswith("prepass")]
step = seq[starts[-1]:]
tot = {}
for k, v in step:
    tot[k] = tot.get(k, 0.0) + v
for k, v in sorted(tot.items(), key=lambda kv: -kv[1])[:20]:
    print(f"{v:8.3f} ms  {k}")
