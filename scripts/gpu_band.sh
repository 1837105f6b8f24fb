# band LU: parity tests, then the factor time at 1 and 2 CTAs per SM
python -m pytest tests/test_gpu_parity.py -q -m gpu -k "band or implicit" 2>&1 | tail -1
for m in 2 1; do echo "minb $m"; LANDAU_BAND_MINB=$m python scripts/band_timing.py 2>&1 | tail -1; done
