python -c "import __graft_entry__ as G; G.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_multi.py -x -q -s > gpurun_out/pytest_multi.log 2>&1
timeout 600 python tools/partition_time.py c2 c4 > gpurun_out/partition_time.txt 2>&1
timeout 900 compute-sanitizer --tool memcheck --leak-check full python tools/sanitize.py > gpurun_out/sanitizer_memcheck.txt 2>&1
timeout 1200 compute-sanitizer --tool racecheck python tools/sanitize.py small > gpurun_out/sanitizer_racecheck.txt 2>&1
timeout 900 compute-sanitizer --tool synccheck python tools/sanitize.py small > gpurun_out/sanitizer_synccheck.txt 2>&1
