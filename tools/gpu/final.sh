# final round-2 check: build, every GPU test, smoke, the default bench line, C5 / C3 / C2 lines, reference arm
python -c "import __graft_entry__ as G; G.build()" > gpurun_out/build.log 2>&1
timeout 2400 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu_all.log 2>&1
timeout 600 python -c "import __graft_entry__ as G; G.smoke()" > gpurun_out/smoke.log 2>&1
timeout 900 python bench.py --steps 20 --warmup 5 > gpurun_out/bench_final_c4.log 2>&1
timeout 900 python bench.py --config c5 --steps 5 --warmup 3 > gpurun_out/bench_final_c5.log 2>&1
timeout 600 python bench.py --config c3 --steps 10 --warmup 3 > gpurun_out/bench_final_c3.log 2>&1
timeout 600 python bench.py --config c2 --steps 10 --warmup 3 > gpurun_out/bench_final_c2.log 2>&1
timeout 600 python bench.py --config c4 --order lex --steps 10 --warmup 3 > gpurun_out/bench_final_c4lex.log 2>&1
timeout 900 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/bench_final_ref.log 2>&1
