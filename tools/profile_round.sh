set -x
timeout 300 python -m pytest tests/test_nsys.py tests/test_gpu_quality.py -q 2>&1 | tail -2
python bench.py 2>gpurun_out/bench_err.log | tail -1 > gpurun_out/r01_bench_c5.json
python bench.py --impl reference --steps 2 --warmup 1 2>/dev/null | tail -1 > gpurun_out/r01_bench_reference.json
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r01_launches_c5.csv python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > /dev/null 2>&1
python tools/launch_summary.py gpurun_out/r01_launches_c5.csv > gpurun_out/r01_launches_c5.txt 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:onesweep -s 2 -c 1 -o gpurun_out/r01_prof_sort_mid_c5 python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"prepass|pm_sums|pm_apply|big_split|small_split|decide|onesweep_kernel<256, 20, true|flag_c|sample_kernel" -c 14 -o gpurun_out/r01_prof_other_c5 python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline > /dev/null 2>&1
ls -la gpurun_out
