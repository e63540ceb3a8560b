#!/bin/bash
# The round's GPU evidence (run under gpurun from the repo root): bench line, reference
# arm, launch list, ncu --set full of the dominant kernel (a middle sort pass), of the
# first sort pass and of the other hot kernels.  Outputs land in gpurun_out/.
set -x
python bench.py 2>gpurun_out/bench_err.log | tail -1 > gpurun_out/r01_bench_c5.json
python bench.py --impl reference --steps 2 --warmup 1 2>/dev/null | tail -1 > gpurun_out/r01_bench_reference.json
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r01_launches_c5.csv \
    python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > /dev/null 2>&1
python tools/launch_summary.py gpurun_out/r01_launches_c5.csv > gpurun_out/r01_launches_c5.txt 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:onesweep -s 2 -c 1 \
    -o gpurun_out/r01_prof_sort_mid_c5 python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:onesweep -s 0 -c 1 \
    -o gpurun_out/r01_prof_sort_first_c5 python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on \
    -k regex:"prepass|pm_sums|pm_apply|big_split|small_split|decide|flag_c|sample_kernel|estimate" -c 16 \
    -o gpurun_out/r01_prof_other_c5 python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline > /dev/null 2>&1
ls -la gpurun_out
