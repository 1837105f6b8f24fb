# band LU: parity tests + timing of both occupancy variants
python -m pytest tests/test_gpu_parity.py -q -m gpu -k "band or more_error" 2>&1 | tail -3
for m in 2 1; do LANDAU_BAND_MINB=$m python scripts/band_timing.py 2>&1 | tail -2; done
