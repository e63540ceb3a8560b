#!/bin/bash
# The round's GPU evidence (run under gpurun from the repo root): bench line, reference
# arm, launch list, ncu --set full of the dominant kernel (a middle sort pass) and of the
# other hot kernels, the split-variant bench lines.  Outputs land in gpurun_out/ with the
# round tag R (default r02).
R=${R:-r02}
set -x
python -c "import __graft_entry__ as g; g.build()"
python bench.py --steps 20 --warmup 5 2>gpurun_out/bench_err.log | tail -1 > gpurun_out/${R}_bench_c5.json
python bench.py --impl reference --steps 2 --warmup 1 2>/dev/null | tail -1 > gpurun_out/${R}_bench_reference.json
for s in 1 2; do
  python bench.py --split $s --steps 10 --warmup 3 --no-e2e --no-cpu-baseline 2>/dev/null | tail -1 > gpurun_out/${R}_bench_c5_split$s.json
done
python bench.py --split 3 --config C3 --steps 5 --warmup 2 --no-e2e --no-cpu-baseline 2>/dev/null | tail -1 > gpurun_out/${R}_bench_c3_kmeans3.json
python bench.py --config C3 --metric-bounds --steps 5 --warmup 2 --no-cpu-baseline 2>/dev/null | tail -1 > gpurun_out/${R}_bench_c3_metric_bounds.json
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${R}_launches_c5.csv \
    python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > /dev/null 2>&1
python tools/launch_summary.py gpurun_out/${R}_launches_c5.csv > gpurun_out/${R}_launches_c5.txt 2>&1
python tools/level_table.py gpurun_out/${R}_launches_c5.csv > gpurun_out/${R}_levels_c5.txt 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:onesweep -s 2 -c 1 \
    -o gpurun_out/${R}_prof_sort_mid_c5 python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on \
    -k regex:"prepass|pm_sums|pm_apply|nc_split|decide|flag_c|sample_kernel|estimate|onesweep" -c 30 \
    -o gpurun_out/${R}_prof_other_c5 python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline > /dev/null 2>&1
# summaries here; only the small reports travel back (gpurun_out must stay under 64 MiB)
python tools/ncu_summary.py gpurun_out/${R}_prof_sort_mid_c5.ncu-rep --traffic-json gpurun_out/ncu_traffic.json --config C5 --stage sort_pass_mid > gpurun_out/${R}_ncu_sort_mid_c5.txt 2>&1
python tools/sass_hot.py gpurun_out/${R}_prof_sort_mid_c5.ncu-rep 25 >> gpurun_out/${R}_ncu_sort_mid_c5.txt 2>&1
python tools/ncu_summary.py gpurun_out/${R}_prof_other_c5.ncu-rep > gpurun_out/${R}_ncu_other_c5.txt 2>&1
python tools/sass_hot.py gpurun_out/${R}_prof_other_c5.ncu-rep 15 nc_split >> gpurun_out/${R}_ncu_other_c5.txt 2>&1
rm -f gpurun_out/${R}_prof_other_c5.ncu-rep
du -sh gpurun_out; ls -la gpurun_out
