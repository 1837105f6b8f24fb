for C in 0 24 48 96; do
LANDAU_CHUNK_MB=$C python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bc.json 2>gpurun_out/bc.err
python -c "import json; d=json.load(open('gpurun_out/bc.json')); print('chunk $C MB', round(d['value']), round(d['ms_per_step'],4), {k: round(v,4) for k,v in d['stage_ms_per_step'].items() if v})" || tail -3 gpurun_out/bc.err
done
