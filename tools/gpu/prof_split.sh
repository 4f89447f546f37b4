# per-visit cycle split of k_prop_async (ECL_PROF builds): all visits, first (full) visits only, later visits only
for sel in all 1 0; do
  if [ $sel = all ]; then X=""; else X="-DECL_PROF_FULL=$sel"; fi
  ECL_PROF=1 ECL_NVCC_EXTRA="$X" python -c "from paper_conf_sc_alabandisbb23_b200 import build as B; B.build(force=True)" > gpurun_out/build_prof_$sel.log 2>&1
  for c in c4 c2; do python tools/prof_one.py $c blocked8 2>&1 | tail -2 > gpurun_out/prof_${c}_$sel.txt; done
done
