for f in build_variants/liblandau_*.so; do
  n=$(basename $f .so)
  LANDAU_LIB=$f python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/b_$n.json 2>gpurun_out/b_$n.err
  python -c "import json; d=json.load(open('gpurun_out/b_$n.json')); print('$n', round(d['value']), 'builds/s inner', round(d['stage_ms_per_step']['inner'],3), 'ms')" || tail -3 gpurun_out/b_$n.err
done
