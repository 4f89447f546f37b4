# compute-sanitizer evidence for the current build (memcheck, synccheck on the full workload; racecheck on the small one)
timeout 1500 compute-sanitizer --tool memcheck --leak-check full python tools/sanitize.py > gpurun_out/sanitizer_memcheck.txt 2>&1
timeout 1200 compute-sanitizer --tool synccheck python tools/sanitize.py > gpurun_out/sanitizer_synccheck.txt 2>&1
timeout 2400 compute-sanitizer --tool racecheck python tools/sanitize.py small > gpurun_out/sanitizer_racecheck.txt 2>&1
