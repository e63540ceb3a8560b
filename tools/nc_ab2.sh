# descent-split variants (compile-time)
python -m pytest tests/test_gpu_parity.py -x -q -k "nearest_centre or big_clusters or worked or tie or edge or configs or mixtures" > gpurun_out/nc4_tests.txt 2>&1; echo rc=$? >> gpurun_out/nc4_tests.txt
bash tools/ab_build.sh "-DSR_NC_MINB=9" "-DSR_NC_MINB=8" "-DSR_NC_MINB=7" > gpurun_out/nc4_ab.txt 2>&1
