python -c "import __graft_entry__ as G; G.build()" > gpurun_out/build.log 2>&1
for c in 148 74 37 16 8; do echo "== ECL_SCC_LV_CTAS=$c"; ECL_SCC_LV_CTAS=$c timeout 300 python tools/levels_time.py c4 c2; done > gpurun_out/levels_ctas.txt 2>&1
