python -m pytest tests/test_gpu_parity.py -q -m gpu -k "band or implicit or newton" 2>&1 | tail -1
python scripts/band_timing.py 2>&1 | tail -1
