ECL_SCC_DEBUG=1 timeout 900 python tools/levels_time.py c5one mesh90 mesh110 > gpurun_out/levels_time3.txt 2>&1
