for n in plain g4 g8; do echo "== $n"; LANDAU_LIB=build_variants/liblandau_sb_$n.so timeout 300 python scripts/c2_latency.py 2>&1 | grep "^SB" | tail -4; done
