# per-visit protocol split of k_prop_async (ECL_PROF + ECL_PROF_PROTO build): claims, visit, fences + marks + finish
ECL_PROF=1 ECL_NVCC_EXTRA="-DECL_PROF_PROTO" python -c "from paper_conf_sc_alabandisbb23_b200 import build as B; B.build(force=True)" > gpurun_out/build_proto.log 2>&1
for c in c4 c2; do PROF_PROTO=1 python tools/prof_one.py $c blocked8 2>&1 | tail -3 > gpurun_out/proto_$c.txt; done
python -c "from paper_conf_sc_alabandisbb23_b200 import build as B; B.build(force=True)" > gpurun_out/build.log 2>&1
timeout 300 python tools/iter_profile.py c4 > gpurun_out/iter_c4_b.txt 2>&1
