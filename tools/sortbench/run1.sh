python tools/sortbench/sortbench.py --check -- "" > gpurun_out/sb1.txt 2>&1
python tools/sortbench/sortbench.py -- "-DSR_SORT_FAKE_LB=1" "-DSR_SORT_FAKE_RANK=1" "-DSR_SORT_FAKE_RANK=1 -DSR_SORT_FAKE_LB=1" >> gpurun_out/sb1.txt 2>&1
