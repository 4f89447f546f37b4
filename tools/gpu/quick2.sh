# quick check: build, parity tests (incl. batched_host), C4 x2 / C2 / C5 (with e2e) bench lines
python -c "import __graft_entry__ as G; G.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "not c5_batched_meshes_full" > gpurun_out/pytest_quick.log 2>&1
for k in 1 2; do timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/q_c4_$k.log 2>&1; done
timeout 300 python bench.py --config c2 --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/q_c2.log 2>&1
timeout 600 python bench.py --config c5 --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/q_c5.log 2>&1
