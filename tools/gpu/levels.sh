# levels: parity (both algorithms) and device time
timeout 900 python -m pytest tests/test_gpu_levels.py -x -q > gpurun_out/pytest_levels.log 2>&1
ECL_SCC_DEBUG=1 timeout 900 python tools/levels_time.py c2 c3 c4 c5one > gpurun_out/levels_time.txt 2>&1
