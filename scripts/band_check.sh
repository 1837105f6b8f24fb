# band LU: parity tests (default = column-warp kernel), factor timing of both kernels in the newton sub-line
timeout 600 python -m pytest tests -m gpu -x -q -k "band or implicit" > gpurun_out/band_tests.log 2>&1
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/band_bench.json 2> gpurun_out/band_bench.err
LANDAU_BAND_CW=0 timeout 600 python bench.py --no-cpu-baseline > gpurun_out/band_bench_old.json 2> gpurun_out/band_bench_old.err
