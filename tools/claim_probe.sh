for c in 1 2 3 4 6 8 16; do echo "CLAIM=$c"; ECL_SCC_CLAIM=$c QT_FLAGS=0 python tools/quick_time.py c2 c4 2>&1 | cut -c1-120; done
