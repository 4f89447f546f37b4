# per-visit cycle split of k_prop_async (ECL_PROF build), C4 blocked8 and C2 blocked8
ECL_PROF=1 python -c "import __graft_entry__ as G; G.build()" > gpurun_out/build_prof.log 2>&1
python tools/prof_one.py c4 blocked8 > gpurun_out/prof_visit_c4.txt 2>&1
python tools/prof_one.py c2 blocked8 > gpurun_out/prof_visit_c2.txt 2>&1
