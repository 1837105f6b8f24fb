for cfg in "12 32" "12 16" "24 16" "24 8" "48 8" "36 8"; do set -- $cfg
  LANDAU_SPLIT_WARPS_PER_SM=$1 LANDAU_SPLIT_MIN=$2 python bench.py --workload C2 --steps 20 --warmup 5 --no-cpu-baseline > gpurun_out/s.json 2>/dev/null
  python -c "import json; d=json.load(open('gpurun_out/s.json')); print('wps $1 min $2', round(d['value']), round(d['ms_per_step']*1e3,1), 'us', {k: round(v*1e3,1) for k,v in d['stage_ms_per_step'].items() if v})"
done
