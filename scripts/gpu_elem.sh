python -m pytest tests/ -x -q -m gpu 2>&1 | tail -2
for SF in 1 0; do
for W in C4 C5 C1; do
  LANDAU_ELEMENT_SF=$SF python bench.py --workload $W --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bench_sf${SF}_$W.json 2> gpurun_out/bench_sf${SF}_$W.err
  python -c "import json; d=json.load(open('gpurun_out/bench_sf${SF}_$W.json')); print('SF=$SF $W', round(d['value']), 'builds/s', round(d['ms_per_step'],3), 'ms', {k: round(v,3) for k,v in d['stage_ms_per_step'].items() if v})" || tail -5 gpurun_out/bench_sf${SF}_$W.err
done; done
