python -c "import __graft_entry__ as G; G.build()" > gpurun_out/build.log 2>&1
for m in 0 2 3; do
  for c in "c4 blocked8" "c4 lex" "c2 blocked8" "c2 lex" "c5 blocked8"; do
    set -- $c
    ECL_SCC_PRIO_MODE=$m timeout 300 python bench.py --config $1 --order $2 --steps 5 --warmup 2 --no-e2e --no-cpu-baseline > gpurun_out/prio_m${m}_$1_$2.log 2>&1
  done
done
for c in "c4 blocked8" "c4 lex" "c2 blocked8" "c5 blocked8"; do set -- $c; timeout 300 python bench.py --config $1 --order $2 --flags 0x20 --steps 5 --warmup 2 --no-e2e --no-cpu-baseline > gpurun_out/prio_ids_$1_$2.log 2>&1; done
