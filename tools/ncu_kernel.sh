#!/bin/bash
# ncu --set full of the kernels matching a regex in one C5 bench step, summarised (run under gpurun)
#   tools/ncu_kernel.sh REGEX COUNT [TAG]   (extra env, e.g. STEMROOT_VALUE_SYNC=1, passes through)
cd "$(dirname "$0")/.."
RE=$1; CNT=${2:-4}; TAG=${3:-k}
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"$RE" -c $CNT \
    -o gpurun_out/prof_$TAG python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline > /dev/null 2>&1
python tools/ncu_summary.py gpurun_out/prof_$TAG.ncu-rep > gpurun_out/ncu_$TAG.txt 2>&1
for k in $(echo "$RE" | tr '|' ' '); do python tools/sass_hot.py gpurun_out/prof_$TAG.ncu-rep 18 "$k" >> gpurun_out/ncu_$TAG.txt 2>&1; done
rm -f gpurun_out/prof_$TAG.ncu-rep
cat gpurun_out/ncu_$TAG.txt
