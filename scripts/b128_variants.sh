for bpt in 4 2 1; do echo "== BPT $bpt"; LANDAU_ASM_BPT=$bpt timeout 300 python bench.py --batch 128 --no-sublines --no-cpu-baseline 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print(round(d['ms_per_step'],4), {k: round(v*1e3,1) for k,v in d['stage_ms_per_step'].items() if v})"; done
