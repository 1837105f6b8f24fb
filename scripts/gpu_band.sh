# band LU: parity tests (both kernels) + timing of the variants
python -m pytest tests/test_gpu_parity.py -q -m gpu -k "band or implicit" 2>&1 | tail -2
LANDAU_BAND_RANK=1 python -m pytest tests/test_gpu_parity.py -q -m gpu -k "band" 2>&1 | tail -1
for r in 2 1; do for m in 2 1; do echo "rank $r minb $m"; LANDAU_BAND_RANK=$r LANDAU_BAND_MINB=$m python scripts/band_timing.py 2>&1 | tail -1; done; done
