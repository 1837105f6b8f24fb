for NI in 2 3; do
  LANDAU_LIB=build_variants/liblandau_ni$NI.so python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/b_ni$NI.json 2>gpurun_out/b_ni$NI.err
  python -c "import json; d=json.load(open('gpurun_out/b_ni$NI.json')); print('NI=$NI', round(d['value']), 'builds/s', round(d['ms_per_step'],3), 'ms', {k: round(v,3) for k,v in d['stage_ms_per_step'].items()})" || tail -3 gpurun_out/b_ni$NI.err
done
