ECL_SCC_DEBUG=1 timeout 900 python tools/levels_time.py c4 c5one > gpurun_out/levels_time2.txt 2>&1
