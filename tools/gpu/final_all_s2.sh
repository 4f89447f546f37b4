# round-2 final run of the current build: every GPU test, smoke, per-config ncu launch lists and a
# full k_prop_async capture, then the bench lines (their traffic field reads the ncu summary committed before this run)
python -c "import __graft_entry__ as G; G.build()" > gpurun_out/build.log 2>&1
timeout 2400 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu_all.log 2>&1
timeout 600 python -c "import __graft_entry__ as G; G.smoke()" > gpurun_out/smoke.log 2>&1
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_requests_srcunit_tex_op_atom.sum,lts__t_requests_srcunit_tex_op_red.sum,lts__t_sector_hit_rate.pct,l1tex__t_sector_hit_rate.pct,sm__warps_active.avg.pct_of_peak_sustained_active,dram__throughput.avg.pct_of_peak_sustained_elapsed
for spec in "c4 blocked8" "c3 x" "c2 blocked8" "c4 lex"; do
  set -- $spec
  timeout 900 ncu --profile-from-start off --clock-control none --metrics $M --csv --log-file gpurun_out/ncu_$1_$2.csv python tools/prof_one.py $1 $2 > gpurun_out/ncu_$1_$2.log 2>&1
done
timeout 1500 ncu --profile-from-start off --clock-control none --metrics $M --csv --log-file gpurun_out/ncu_c5_blocked8.csv python tools/prof_one_c5.py > gpurun_out/ncu_c5.log 2>&1
timeout 900 ncu --profile-from-start off --set full --clock-control none --import-source on -k regex:k_prop_async -c 1 -o gpurun_out/full_c4 python tools/prof_one.py c4 blocked8 > gpurun_out/full_c4.log 2>&1
timeout 900 python bench.py --steps 20 --warmup 5 > gpurun_out/bench_final_c4.log 2>&1
timeout 1200 python bench.py --config c5 --steps 5 --warmup 3 > gpurun_out/bench_final_c5.log 2>&1
timeout 600 python bench.py --config c3 --steps 10 --warmup 3 > gpurun_out/bench_final_c3.log 2>&1
timeout 600 python bench.py --config c2 --steps 10 --warmup 3 > gpurun_out/bench_final_c2.log 2>&1
timeout 600 python bench.py --config c4 --order lex --steps 10 --warmup 3 > gpurun_out/bench_final_c4lex.log 2>&1
timeout 900 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/bench_final_ref.log 2>&1
timeout 600 python tools/iter_profile.py c4 > gpurun_out/iter_final_c4.txt 2>&1
timeout 600 python tools/levels_time.py > gpurun_out/levels_final.txt 2>&1
timeout 900 python tools/partition_time.py > gpurun_out/partition_emulated_final.txt 2>&1
