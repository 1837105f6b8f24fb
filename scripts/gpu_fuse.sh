python -m pytest tests/ -x -q -m gpu 2>&1 | tail -2
for F in 1 0; do for i in 1 2; do
LANDAU_FUSE_FE=$F python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bf.json 2>gpurun_out/bf.err
python -c "import json; d=json.load(open('gpurun_out/bf.json')); print('fuse $F', round(d['value']), round(d['ms_per_step'],4), {k: round(v,4) for k,v in d['stage_ms_per_step'].items() if v}, 'e2e', round(d['e2e']['value']), 'newton', round(d['newton']['value']))" || tail -3 gpurun_out/bf.err
done; done
