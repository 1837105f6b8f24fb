python -m pytest tests/ -x -q -m gpu 2>&1 | tail -2
for W in C4 C5 C2; do
  python bench.py --workload $W --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bench_q_$W.json 2> gpurun_out/bench_q_$W.err
  python -c "import json; d=json.load(open('gpurun_out/bench_q_$W.json')); print('$W', round(d['value']), 'builds/s', round(d['ms_per_step'],4), 'ms', {k: round(v,4) for k,v in d['stage_ms_per_step'].items() if v})" || tail -5 gpurun_out/bench_q_$W.err
done
