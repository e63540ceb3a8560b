# descent-split variants (compile-time) and the sort's first-pass publication mode
python -m pytest tests/test_gpu_parity.py tests/test_gpu_dist.py -x -q > gpurun_out/nc3_tests.txt 2>&1; echo rc=$? >> gpurun_out/nc3_tests.txt
bash tools/ab_build.sh "-DSR_NC_SBEST=0" "-DSR_NC_SBEST=1" "-DSR_NC_SBEST=1 -DSR_NC_THREADS=128 -DSR_NC_MINB=9" > gpurun_out/nc3_ab.txt 2>&1
python tools/sortbench/sortbench.py -- "" > gpurun_out/sb3.txt 2>&1
STEMROOT_SORT_LATE_FIRST=0 python tools/sortbench/sortbench.py -- "" >> gpurun_out/sb3.txt 2>&1
