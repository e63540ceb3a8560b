python -m pytest tests/test_gpu_parity.py -x -q -k "nearest_centre" > gpurun_out/nc_tests.txt 2>&1; echo rc=$? >> gpurun_out/nc_tests.txt
bash tools/ab.sh "STEMROOT_SPLIT_NC=0" "STEMROOT_SPLIT_NC=1" "STEMROOT_SPLIT_NC=2" "STEMROOT_SPLIT_NC=2 STEMROOT_VALUE_ROWS=0" "STEMROOT_SPLIT_NC=0" > gpurun_out/nc_ab.txt 2>&1
