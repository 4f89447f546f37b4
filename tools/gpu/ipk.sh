timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_variants.py -x -q > gpurun_out/pytest_quick.log 2>&1
for k in 80 101; do ECL_SCC_IP_KEEP=$k timeout 600 python tools/iter_profile.py c4 > gpurun_out/iter_ipk_$k.txt 2>&1; done
for k in 80 101; do
ECL_SCC_IP_KEEP=$k timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/q_c4_ipk$k.log 2>&1
ECL_SCC_IP_KEEP=$k timeout 300 python bench.py --config c4 --order lex --steps 5 --warmup 2 --no-e2e --no-cpu-baseline > gpurun_out/q_c4lex_ipk$k.log 2>&1
ECL_SCC_IP_KEEP=$k timeout 300 python bench.py --config c5 --steps 3 --warmup 2 --no-e2e --no-cpu-baseline > gpurun_out/q_c5_ipk$k.log 2>&1
done
