python -m pytest tests/ -x -q -m gpu 2>&1 | tail -3
for B in 1024 512 256 148 128; do
  python bench.py --batch $B --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bench_h_${B}.json 2> gpurun_out/bench_h_${B}.err
  python -c "import json; d=json.load(open('gpurun_out/bench_h_${B}.json')); print('B=$B', round(d['value']), 'builds/s', round(d['ms_per_step'],3), 'ms', {k: round(v,3) for k,v in d['stage_ms_per_step'].items() if v}, 'frac', round(d['roofline']['frac'],3), d['roofline']['inner_path'])" || tail -5 gpurun_out/bench_h_${B}.err
done
