for cfg in "12 32" "12 16" "12 8" "24 8" "24 4"; do set -- $cfg
for W in C2 C3; do
LANDAU_MDIR_WARPS_PER_SM=$1 LANDAU_MDIR_SPLIT_MIN=$2 python bench.py --workload $W --steps 20 --warmup 5 --no-cpu-baseline > gpurun_out/bm.json 2>gpurun_out/bm.err
python -c "import json; d=json.load(open('gpurun_out/bm.json')); print('$W wps $1 min $2', round(d['value']), round(d['ms_per_step']*1e3,1), 'us', {k: round(v*1e3,1) for k,v in d['stage_ms_per_step'].items() if v})" || tail -3 gpurun_out/bm.err
done; done
