python -m pytest tests/ -x -q -m gpu 2>&1 | tail -1
for A in 1 0; do for i in 1 2; do
LANDAU_ASM_WARP=$A python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/ba.json 2>gpurun_out/ba.err
python -c "import json; d=json.load(open('gpurun_out/ba.json')); print('asm_warp $A', round(d['value']), round(d['ms_per_step'],4), {k: round(v,4) for k,v in d['stage_ms_per_step'].items() if v})" || tail -3 gpurun_out/ba.err
done; done
