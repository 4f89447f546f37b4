set -x
python -c "import __graft_entry__ as G; G.build()" > gpurun_out/build.log 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1
timeout 600 python bench.py --steps 10 --warmup 3 > gpurun_out/bench_c4.log 2>&1
timeout 600 python bench.py --config c5 --steps 5 --warmup 3 > gpurun_out/bench_c5.log 2>&1
