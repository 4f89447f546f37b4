# quick check of a Phase-2 change: build, parity + variants tests, C4/C2/C5 bench lines (device time only)
# (prebuilt library)
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_variants.py -x -q > gpurun_out/pytest_quick.log 2>&1
for k in 1 2; do timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/q_c4_$k.log 2>&1; done
timeout 300 python bench.py --config c4 --order lex --steps 5 --warmup 2 --no-e2e --no-cpu-baseline > gpurun_out/q_c4lex.log 2>&1
timeout 300 python bench.py --config c2 --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/q_c2.log 2>&1
timeout 300 python bench.py --config c5 --steps 3 --warmup 2 --no-e2e --no-cpu-baseline > gpurun_out/q_c5.log 2>&1
