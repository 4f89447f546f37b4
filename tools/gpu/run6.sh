python -c "import __graft_entry__ as G; G.build()" > gpurun_out/build.log 2>&1
timeout 600 python tools/partition_time.py c2 c4 > gpurun_out/partition_time.txt 2>&1
timeout 600 python tools/iter_profile.py c4 c2 c3 > gpurun_out/iter_profile.txt 2>&1
timeout 600 python bench.py --gpus 1 --config c4 --steps 3 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/bench_smoke.log 2>&1
