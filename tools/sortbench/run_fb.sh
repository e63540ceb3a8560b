for fb in 3 4 2; do echo "FIRST_BLOCKS=$fb"; STEMROOT_FIRST_BLOCKS=$fb python tools/sortbench/sortbench.py -- "" ; done > gpurun_out/fb.txt 2>&1
