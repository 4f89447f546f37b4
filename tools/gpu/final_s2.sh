# round-2 final bench lines (current build, after the ncu summaries of evidence_s2.sh are committed):
# C4 (the default line), C5 (with the batched host-buffer e2e), C3, C2, C4 lex, the reference arm,
# per-iteration split, levels and emulated-partition timings
python -c "import __graft_entry__ as G; G.build()" > gpurun_out/build.log 2>&1
timeout 900 python bench.py --steps 20 --warmup 5 > gpurun_out/bench_final_c4.log 2>&1
timeout 1200 python bench.py --config c5 --steps 5 --warmup 3 > gpurun_out/bench_final_c5.log 2>&1
timeout 600 python bench.py --config c3 --steps 10 --warmup 3 > gpurun_out/bench_final_c3.log 2>&1
timeout 600 python bench.py --config c2 --steps 10 --warmup 3 > gpurun_out/bench_final_c2.log 2>&1
timeout 600 python bench.py --config c4 --order lex --steps 10 --warmup 3 > gpurun_out/bench_final_c4lex.log 2>&1
timeout 900 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/bench_final_ref.log 2>&1
timeout 600 python tools/iter_profile.py c4 > gpurun_out/iter_final_c4.txt 2>&1
timeout 600 python tools/levels_time.py > gpurun_out/levels_final.txt 2>&1
timeout 900 python tools/partition_time.py > gpurun_out/partition_emulated_final.txt 2>&1
