for F in 8 16 32 1000; do
LANDAU_FIELD_BLOCKS_PER_SM=$F python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bf.json 2>gpurun_out/bf.err
python -c "import json; d=json.load(open('gpurun_out/bf.json')); print('field bps $F', round(d['value']), round(d['ms_per_step'],4), {k: round(v,4) for k,v in d['stage_ms_per_step'].items() if v})" || tail -3 gpurun_out/bf.err
done
