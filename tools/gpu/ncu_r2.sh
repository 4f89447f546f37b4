# round-2 ncu evidence: per config one ecl_scc run (launch list with DRAM bytes, L2 atomics,
# hit rates) and a full capture of the dominant Phase-2 kernel
python -c "import __graft_entry__ as G; G.build()" > gpurun_out/build.log 2>&1
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_requests_srcunit_tex_op_atom.sum,lts__t_requests_srcunit_tex_op_red.sum,lts__t_sector_hit_rate.pct,l1tex__t_sector_hit_rate.pct,sm__warps_active.avg.pct_of_peak_sustained_active,dram__throughput.avg.pct_of_peak_sustained_elapsed
for spec in "c4 blocked8" "c3 x" "c2 blocked8" "c4 lex"; do
  set -- $spec
  timeout 900 ncu --profile-from-start off --clock-control none --metrics $M --csv --log-file gpurun_out/ncu_$1_$2.csv python tools/prof_one.py $1 $2 > gpurun_out/ncu_$1_$2.log 2>&1
done
timeout 900 ncu --profile-from-start off --set full --clock-control none --import-source on -k regex:k_prop_async -c 1 -o gpurun_out/full_c4 python tools/prof_one.py c4 blocked8 > gpurun_out/full_c4.log 2>&1
timeout 900 ncu --profile-from-start off --set full --clock-control none --import-source on -k regex:k_prop_tile -c 1 -o gpurun_out/full_c3 python tools/prof_one.py c3 x > gpurun_out/full_c3.log 2>&1
timeout 900 ncu --profile-from-start off --set full --clock-control none --import-source on -k regex:k_compact_scatter -s 1 -c 1 -o gpurun_out/full_c4_scatter python tools/prof_one.py c4 blocked8 > gpurun_out/full_c4_scatter.log 2>&1
