# C2 single build: set_state + jacobian time with phases of the fused kernel skipped (build variants,
# results wrong by construction; measures each phase's in-situ cost)
for m in 0 1 2 4 8 16 31; do echo "== skip $m"; LANDAU_LIB=build_variants/liblandau_skip$m.so timeout 300 python scripts/c2_latency.py 2>&1 | grep "C2 graph"; done
