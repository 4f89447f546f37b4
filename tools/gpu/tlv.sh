# tile level schedule (ECL_SCC_TLV=2) vs flags-only drain (=1) vs schedule built but unused (=3)
python -c "import __graft_entry__ as G; G.build()" > gpurun_out/build.log 2>&1
ECL_SCC_TLV=2 timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_variants.py -x -q > gpurun_out/pytest_tlv.log 2>&1
for t in 1 2 3; do
  ECL_SCC_TLV=$t timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/tlv${t}_c4.log 2>&1
  ECL_SCC_TLV=$t timeout 300 python bench.py --config c2 --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/tlv${t}_c2.log 2>&1
done
for t in 1 2; do
  ECL_SCC_TLV=$t timeout 300 python bench.py --config c4 --order lex --steps 5 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/tlv${t}_c4lex.log 2>&1
  ECL_SCC_TLV=$t timeout 300 python bench.py --config c5 --steps 3 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/tlv${t}_c5.log 2>&1
done
ECL_SCC_TLV=2 timeout 300 python tools/iter_profile.py c4 > gpurun_out/iter_tlv2_c4.txt 2>&1
for sel in all 1 0; do
  if [ $sel = all ]; then X=""; else X="-DECL_PROF_FULL=$sel"; fi
  ECL_PROF=1 ECL_NVCC_EXTRA="$X" python -c "from paper_conf_sc_alabandisbb23_b200 import build as B; B.build(force=True)" > gpurun_out/build_prof_$sel.log 2>&1
  ECL_SCC_TLV=2 python tools/prof_one.py c4 blocked8 2>&1 | tail -3 > gpurun_out/tprof_c4_$sel.txt
done
