python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "band or implicit" 2>&1 | tail -1
for f in paper_conf_ipps_adamsbkw22_b200/liblandau.so build_variants/liblandau_kb8.so build_variants/liblandau_kb2.so; do echo $f; LANDAU_LIB=$f python scripts/band_timing.py 2>&1 | tail -1; done
