# ncu: per-kernel times of one C4 run and a full capture of the keep-word compaction count / scatter
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,sm__inst_executed.sum,lts__t_sector_hit_rate.pct
timeout 900 ncu --profile-from-start off --clock-control none --metrics $M --csv --log-file gpurun_out/ncu_c4_kw.csv python tools/prof_one.py c4 blocked8 > gpurun_out/ncu_c4_kw.log 2>&1
timeout 900 ncu --profile-from-start off --set full --clock-control none --import-source on -k regex:k_compact_count -s 1 -c 1 -o gpurun_out/full_c4_count python tools/prof_one.py c4 blocked8 > gpurun_out/full_c4_count.log 2>&1
timeout 900 ncu --profile-from-start off --set full --clock-control none --import-source on -k regex:k_compact_scatter -s 1 -c 1 -o gpurun_out/full_c4_scatter2 python tools/prof_one.py c4 blocked8 > gpurun_out/full_c4_scatter2.log 2>&1
