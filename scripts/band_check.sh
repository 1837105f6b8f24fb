timeout 600 python -m pytest tests -m gpu -x -q -k "band or implicit" > gpurun_out/band_tests.log 2>&1
python -c "
from paper_conf_ipps_adamsbkw22_b200 import inputs, landau as L
h = L.Landau.from_problem(inputs.config2(), device=0); print('C2 band', h.band_info(0)[0])
" > gpurun_out/band_B.log 2>&1
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/band_bench.json 2> gpurun_out/band_bench.err
