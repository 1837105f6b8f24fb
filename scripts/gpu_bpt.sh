for B in 4 2 1 8; do
LANDAU_ASM_BPT=$B python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bb.json 2>gpurun_out/bb.err
python -c "import json; d=json.load(open('gpurun_out/bb.json')); print('bpt $B', round(d['value']), round(d['ms_per_step'],4), {k: round(v,4) for k,v in d['stage_ms_per_step'].items() if v})" || tail -3 gpurun_out/bb.err
done
