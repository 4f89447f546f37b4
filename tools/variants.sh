#!/bin/bash
# Build and time compile-time variants of the Phase-2 kernels (development helper).
# usage: tools/variants.sh "label1:-DFLAG1 -DFLAG2" "label2:" ...   (run on the GPU box)
for spec in "$@"; do
  label="${spec%%:*}"; flags="${spec#*:}"
  echo "=== variant $label ($flags)"
  ECL_NVCC_EXTRA="$flags -DECL_VARIANT" python -c "from paper_conf_sc_alabandisbb23_b200 import build as B; B.build(force=True)" || continue
  ECL_SCC_DEBUG=1 timeout 300 python tools/iter_profile.py ${VARIANT_CFGS:-c4 c2} 2>&1 | grep -E "==|CTAs per SM" | sort -u
done
