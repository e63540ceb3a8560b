#!/bin/bash
# A/B of the value-histogram ROOT path on the C5 bench: off, concurrent (thresholds), synchronous (timed stage)
cd "$(dirname "$0")/.."
run() { echo "== $1"; env $2 timeout 300 python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu-baseline 2>&1 | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); s=d['stages_ms_per_step']
print(round(d['ms_per_step'],2), {k: round(v,3) for k,v in s.items() if k.startswith('root')})"; }
for cfg in ${VALUE_AB:-"off:STEMROOT_VALUE_ROWS=0" "conc:STEMROOT_VALUE_ROWS=262144" "sync:STEMROOT_VALUE_ROWS=262144,STEMROOT_VALUE_SYNC=1"}; do
  run "${cfg%%:*}" "$(echo ${cfg#*:} | tr , ' ')"
done
