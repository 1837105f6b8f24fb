python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "band or implicit" 2>&1 | tail -2
for R in 4 2; do echo "rank $R"; LANDAU_BAND_RANK=$R python scripts/band_timing.py 2>&1 | tail -1; done
LANDAU_BAND_RANK=2 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "band or implicit" 2>&1 | tail -1
