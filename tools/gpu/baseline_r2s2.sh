# session re-entry check: build, parity tests, C4/C5 bench lines, per-iteration split of C4
python -c "import __graft_entry__ as G; G.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q > gpurun_out/pytest_quick.log 2>&1
for k in 1 2; do timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/q_c4_$k.log 2>&1; done
timeout 300 python bench.py --config c5 --steps 3 --warmup 2 --no-e2e --no-cpu-baseline > gpurun_out/q_c5.log 2>&1
timeout 300 python tools/iter_profile.py c4 > gpurun_out/iter_c4.txt 2>&1
