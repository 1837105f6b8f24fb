timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/vtx_order_tests.log 2>&1
for nb in 128 1024; do echo "== batch $nb"; timeout 300 python bench.py --batch $nb --no-sublines --no-cpu-baseline 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print(round(d['ms_per_step'],4), {k: round(v*1e3,1) for k,v in d['stage_ms_per_step'].items() if v})"; done
