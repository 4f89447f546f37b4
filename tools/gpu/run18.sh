python -c "import __graft_entry__ as G; G.build()" > gpurun_out/build.log 2>&1
timeout 600 python -m pytest tests/test_gpu_multi.py -x -q -s -k "probe or nccl" > gpurun_out/pytest_probe.log 2>&1
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_requests_srcunit_tex_op_atom.sum,lts__t_requests_srcunit_tex_op_red.sum,lts__t_sector_hit_rate.pct,l1tex__t_sector_hit_rate.pct,sm__warps_active.avg.pct_of_peak_sustained_active,dram__throughput.avg.pct_of_peak_sustained_elapsed
timeout 1500 ncu --profile-from-start off --clock-control none --metrics $M --csv --log-file gpurun_out/ncu_c5_blocked8.csv python tools/prof_one_c5.py > gpurun_out/ncu_c5.log 2>&1
