#!/bin/bash
# tile-size sweep on C4/C2 (development helper); prof counters need an ECL_PROF build
for t in 512 1024 2048 4096; do
  ECL_SCC_TILE=$t python tools/quick_time.py $@ 2>&1 | sed "s/^/tile=$t /"
done
