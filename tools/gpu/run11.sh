python -c "import __graft_entry__ as G; G.build()" > gpurun_out/build.log 2>&1
timeout 600 python -m pytest tests/test_gpu_variants.py -x -q -k cluster > gpurun_out/pytest_cluster.log 2>&1
for f in 0 0x40000; do
  timeout 300 python bench.py --config c4 --flags $f --steps 5 --warmup 2 --no-e2e --no-cpu-baseline > gpurun_out/bench_c4_f$f.log 2>&1
  timeout 300 python bench.py --config c2 --flags $f --steps 5 --warmup 2 --no-e2e --no-cpu-baseline > gpurun_out/bench_c2_f$f.log 2>&1
done
