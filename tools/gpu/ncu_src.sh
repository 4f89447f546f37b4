# full ncu captures with source of the compaction kernels (second launch, C4 blocked8) and of
# k_prop_async (first launch); read back here with --page source / details
python -c "import __graft_entry__ as G; G.build()" > gpurun_out/build.log 2>&1
for k in k_compact_scatter k_compact_count k_compact_map k_keep_count; do
  timeout 600 ncu --profile-from-start off --set full --clock-control none --import-source on -k regex:$k -s 1 -c 1 -o gpurun_out/src_$k python tools/prof_one.py c4 blocked8 > gpurun_out/src_$k.log 2>&1
done
timeout 900 ncu --profile-from-start off --set full --clock-control none --import-source on -k regex:k_prop_async -c 1 -o gpurun_out/src_k_prop_async python tools/prof_one.py c4 blocked8 > gpurun_out/src_k_prop_async.log 2>&1
