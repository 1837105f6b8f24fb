python -m pytest tests/ -x -q -m gpu 2>&1 | tail -2
python bench.py --workload C5 --steps 3 --warmup 2 --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('C5', d['value'], d['ms_per_step'], d['roofline']['frac'], d['stage_ms_per_step'])"
