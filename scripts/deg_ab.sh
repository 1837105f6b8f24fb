# same-box A/B: HEAD (degree-10 D fit) vs the working tree (degree-9 D fit)
timeout 900 python -m pytest tests -m gpu -x -q -k "parity or C2 or C1 or C3 or C4 or headline or conservation or stress" > gpurun_out/deg_tests.log 2>&1
for rep in 1 2; do for lib in head d9; do for nb in 128 1024; do echo -n "$lib $nb "; if [ $lib = head ]; then B=build_variants/headpkg/bench.py; else B=bench.py; fi; timeout 300 python $B --batch $nb --steps 30 --no-sublines --no-cpu-baseline 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print(round(d['ms_per_step'],4), round(d['stage_ms_per_step']['inner']*1e3,1))"; done; done; done
timeout 600 python tools/parity_report.py > gpurun_out/deg_parity.json 2>&1
