# mirror-directed split-j sweep (LANDAU_MDIR_SPLIT_MIN) on the single-build configs with the
# split-parallel reduce_mdir_kernel
for m in 16 12 8 6 4; do for w in C2 C3; do echo "min=$m $w"; LANDAU_MDIR_SPLIT_MIN=$m python bench.py --workload $w --steps 20 --warmup 5 --no-cpu-baseline 2>/dev/null | python -c "import json,sys;d=json.loads(sys.stdin.read().strip().splitlines()[-1]);s=d['stage_ms_per_step'];print(round(d['value']),round(d['ms_per_step']*1e3,1),'inner',round(s['inner']*1e3,1),'reduce',round(s['reduce']*1e3,1))"; done; done
