timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/heavy_tests.log 2>&1
for hv in 1 0; do for nb in 128 1024; do echo -n "heavy $hv batch $nb: "; LANDAU_ASM_HEAVY=$hv timeout 300 python bench.py --batch $nb --steps 30 --no-sublines --no-cpu-baseline 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print(round(d['ms_per_step'],4), {k: round(v*1e3,1) for k,v in d['stage_ms_per_step'].items() if v})"; done; done
