# claim-size cap sweep on C5 / C4 (env knob ECL_SCC_CLAIM_MAX; default 16)
python -c "import __graft_entry__ as G; G.build()" > gpurun_out/build.log 2>&1
for cm in 16 32 8; do
  ECL_SCC_CLAIM_MAX=$cm timeout 300 python bench.py --config c5 --steps 3 --warmup 2 --no-e2e --no-cpu-baseline > gpurun_out/cm${cm}_c5.log 2>&1
  ECL_SCC_CLAIM_MAX=$cm timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/cm${cm}_c4.log 2>&1
done
