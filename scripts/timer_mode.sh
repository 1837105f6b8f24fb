for B in 1024 128; do for M in loop separate; do
timeout 300 python bench.py --batch $B --no-sublines --no-cpu-baseline --stage-timers $M 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('B$B $M', round(d['value']), round(d['ms_per_step'],4), round(d['roofline']['frac'],3), {k: round(v,4) for k,v in d['stage_ms_per_step'].items() if v})"
done; done
