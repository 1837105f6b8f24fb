# fused single build: parity tests, phase profile (build variant), C2 bench line
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/sb_tests.log 2>&1
LANDAU_LIB=build_variants/liblandau_sbprof.so timeout 300 python scripts/c2_latency.py > gpurun_out/c2_sbprof.log 2>&1
timeout 300 python scripts/c2_latency.py > gpurun_out/c2_latency.log 2>&1
for W in C1 C2 C3; do timeout 300 python bench.py --workload $W --no-cpu-baseline > gpurun_out/sb_bench_$W.json 2>/dev/null; done
