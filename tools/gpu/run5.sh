python -c "import __graft_entry__ as G; G.build()" > gpurun_out/build.log 2>&1
timeout 1200 python -m pytest tests/test_gpu_multi.py -x -q -s > gpurun_out/pytest_multi.log 2>&1
timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/bench_c4.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q > gpurun_out/pytest_parity.log 2>&1
