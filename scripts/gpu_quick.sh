# quick GPU iteration: parity + C4 bench for both inner-kernel variants
python -m pytest tests/test_gpu_parity.py -x -q -m gpu 2>&1 | tail -3
for T in 1 2; do
  LANDAU_INNER_TPT=$T python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bench_tpt$T.json 2> gpurun_out/bench_tpt$T.err
  python -c "import json; d=json.load(open('gpurun_out/bench_tpt$T.json')); print('TPT=$T', round(d['value']), 'builds/s', round(d['ms_per_step'],3), 'ms', d['stage_ms_per_step'], 'frac', round(d['roofline']['frac'],3), 'e2e', round(d['e2e']['value']))" || tail -5 gpurun_out/bench_tpt$T.err
done
