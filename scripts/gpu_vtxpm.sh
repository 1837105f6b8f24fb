python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "vertex or symmetric or coincident" 2>&1 | tail -2
for i in 1 2; do python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bench_pm.json 2>gpurun_out/bench_pm.err
python -c "import json; d=json.load(open('gpurun_out/bench_pm.json')); print(round(d['value']), 'builds/s', round(d['ms_per_step'],4), 'ms', {k: round(v,4) for k,v in d['stage_ms_per_step'].items() if v}, 'frac', round(d['roofline']['frac'],3))" || tail -3 gpurun_out/bench_pm.err; done
