python -m pytest tests/ -x -q -m gpu 2>&1 | tail -2
LANDAU_VTX_MIN_BATCH_PER_SM=100000 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/b1.json 2>gpurun_out/b1.err
python -c "import json; d=json.load(open('gpurun_out/b1.json')); print('C4 slots', round(d['value']), round(d['ms_per_step'],4), {k: round(v,4) for k,v in d['stage_ms_per_step'].items() if v})" || tail -3 gpurun_out/b1.err
python bench.py --batch 128 --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/b2.json 2>gpurun_out/b2.err
python -c "import json; d=json.load(open('gpurun_out/b2.json')); print('B128', round(d['value']), round(d['ms_per_step'],4), {k: round(v,4) for k,v in d['stage_ms_per_step'].items() if v})" || tail -3 gpurun_out/b2.err
python bench.py --workload C5 --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/b3.json 2>gpurun_out/b3.err
python -c "import json; d=json.load(open('gpurun_out/b3.json')); print('C5', round(d['value'],2), round(d['ms_per_step'],4), {k: round(v,4) for k,v in d['stage_ms_per_step'].items() if v})" || tail -3 gpurun_out/b3.err
