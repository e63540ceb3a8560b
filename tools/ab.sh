#!/bin/bash
# A/B the C5 bench under environment settings: tools/ab.sh "ENV=1 ENV2=0" "ENV=2" ...
# prints ms/step and the per-stage ms for each setting (device time, no e2e / cpu baseline)
for cfg in "$@"; do
  out=$(env $cfg python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu-baseline 2>&1 | tail -1)
  python - "$cfg" "$out" <<'PY'
import json, sys
cfg, line = sys.argv[1], sys.argv[2]
try:
    d = json.loads(line)
except Exception:
    print(cfg, "FAILED:", line[-300:]); sys.exit()
st = " ".join(f"{k}={v:.2f}" for k, v in list(d["stages_ms_per_step"].items())[:9])
print(f"[{cfg}] {d['ms_per_step']:.2f} ms | {st}")
PY
done
