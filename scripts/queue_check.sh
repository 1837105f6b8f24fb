python scripts/vtx_overhead.py
for B in 1024 128; do
timeout 300 python bench.py --batch $B --no-sublines --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('B$B', round(d['value']), round(d['ms_per_step'],4), round(d['roofline']['frac'],3), {k: round(v,4) for k,v in d['stage_ms_per_step'].items() if v})"
done
timeout 900 python -m pytest tests/ -x -q -m gpu 2>&1 | tail -3
