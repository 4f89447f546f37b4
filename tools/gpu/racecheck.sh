timeout 2400 compute-sanitizer --tool racecheck python tools/sanitize.py small > gpurun_out/sanitizer_racecheck.txt 2>&1
