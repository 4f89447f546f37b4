# round-2 final bench lines (current build): default C4 line (e2e + cpu baseline), C5 / C3 / C2 / C4 lex, reference arm
timeout 900 python bench.py --steps 20 --warmup 5 > gpurun_out/bench_final_c4.log 2>&1
timeout 900 python bench.py --config c5 --steps 5 --warmup 3 > gpurun_out/bench_final_c5.log 2>&1
timeout 600 python bench.py --config c3 --steps 10 --warmup 3 > gpurun_out/bench_final_c3.log 2>&1
timeout 600 python bench.py --config c2 --steps 10 --warmup 3 > gpurun_out/bench_final_c2.log 2>&1
timeout 600 python bench.py --config c4 --order lex --steps 10 --warmup 3 > gpurun_out/bench_final_c4lex.log 2>&1
timeout 900 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/bench_final_ref.log 2>&1
timeout 900 python tools/levels_time.py c2 c3 c4 c5one > gpurun_out/levels_time_final.txt 2>&1
