# level-pass profile (ECL_PROF): all / full / non-full visits, C4 and C2
for sel in all 1 0; do
  if [ $sel = all ]; then X=""; else X="-DECL_PROF_FULL=$sel"; fi
  ECL_PROF=1 ECL_NVCC_EXTRA="$X" python -c "from paper_conf_sc_alabandisbb23_b200 import build as B; B.build(force=True)" > gpurun_out/build_prof_$sel.log 2>&1
  for c in c4 c2; do ECL_SCC_TLV=2 python tools/prof_one.py $c blocked8 2>&1 | tail -3 > gpurun_out/tprof_${c}_$sel.txt; done
done
