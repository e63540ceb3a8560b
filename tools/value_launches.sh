#!/bin/bash
# launch list of the value path (synchronous mode) on the C5 bench: per-kernel sums
cd "$(dirname "$0")/.."
STEMROOT_VALUE_SYNC=1 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/vl.csv \
  python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline > /dev/null 2>&1
python - <<PY
import csv, re, collections
rows = [r for r in csv.reader(open("gpurun_out/vl.csv")) if len(r) > 10]
h = rows[0]; ki = h.index("Kernel Name"); vi = h.index("Metric Value")
agg = collections.OrderedDict()
for r in rows[1:]:
    n = re.sub(r"\(.*", "", r[ki].replace("sr::", "").replace("void ", ""))
    a = agg.setdefault(n, [0, 0.0]); a[0] += 1; a[1] += float(r[vi].replace(",", "")) / 1e6
for k, v in sorted(agg.items(), key=lambda kv: -kv[1][1])[:24]:
    print(f"{v[1]:8.3f} ms {v[0]:5d}  {k[:90]}")
PY
rm -f gpurun_out/vl.csv
