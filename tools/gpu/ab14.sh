# A/B: scan top folded into the apply (new) vs three scan kernels (old)
python -c "import __graft_entry__ as G; G.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_variants.py -x -q -k "not c5_batched_meshes_full"; timeout 900 python -m pytest tests/test_gpu_multi.py tests/test_gpu_levels.py -x -q > gpurun_out/pytest_multi.log 2>&1 > gpurun_out/pytest_quick.log 2>&1
for r in 1 2; do
  for v in new old; do
    if [ $v = old ]; then ECL_NVCC_EXTRA="-DECL_AB_OLD" python -c "from paper_conf_sc_alabandisbb23_b200 import build as B; B.build(force=True)" > gpurun_out/build_$v.log 2>&1;
    else python -c "from paper_conf_sc_alabandisbb23_b200 import build as B; B.build(force=True)" > gpurun_out/build_$v.log 2>&1; fi
    timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/ab14_${v}_c4_$r.log 2>&1
    timeout 300 python bench.py --config c2 --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/ab14_${v}_c2_$r.log 2>&1
    timeout 300 python bench.py --config c5 --steps 3 --warmup 2 --no-e2e --no-cpu-baseline > gpurun_out/ab14_${v}_c5_$r.log 2>&1
  done
done
