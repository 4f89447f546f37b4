python -c "import __graft_entry__ as G; G.build()" > gpurun_out/build.log 2>&1
for k in 1 2; do timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/bench_c4_ns_$k.log 2>&1; done
timeout 300 python bench.py --config c2 --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/bench_c2_ns.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_variants.py -x -q > gpurun_out/pytest_ns.log 2>&1
