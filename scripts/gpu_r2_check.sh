# round 2: GPU tests + batch-size sweep of the stream-K per-vertex kernel
set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 900 python -m pytest tests/ -x -q -m gpu 2>&1 | tail -15
for B in 1024 512 256 128 64 37; do
  timeout 300 python bench.py --batch $B --steps 10 --warmup 3 --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('B$B', round(d['value']), round(d['ms_per_step'],4), d['roofline']['inner_path'], round(d['roofline']['frac'],3), {k: round(v,4) for k,v in d['stage_ms_per_step'].items() if v})"
done
