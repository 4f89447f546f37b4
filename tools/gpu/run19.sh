ECL_NVCC_EXTRA="-DECL_DRAIN_STEAL" python -c "from paper_conf_sc_alabandisbb23_b200 import build as B; B.build(force=True)" > gpurun_out/build.log 2>&1
for k in 1 2; do timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/bench_c4_steal_$k.log 2>&1; done
timeout 300 python bench.py --config c2 --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/bench_c2_steal.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q > gpurun_out/pytest_steal.log 2>&1
python -c "from paper_conf_sc_alabandisbb23_b200 import build as B; B.build(force=True)" >> gpurun_out/build.log 2>&1
timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/bench_c4_base.log 2>&1
