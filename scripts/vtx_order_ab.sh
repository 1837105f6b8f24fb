# same-box A/B: HEAD package (build_variants/headpkg) vs the working tree
for rep in 1 2 3; do for lib in head ord; do for nb in 128 1024; do echo -n "$lib $nb "; if [ $lib = head ]; then B=build_variants/headpkg/bench.py; else B=bench.py; fi; timeout 300 python $B --batch $nb --steps 30 --no-sublines --no-cpu-baseline 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print(round(d['ms_per_step'],4), round(d['stage_ms_per_step']['inner']*1e3,1))"; done; done; done
