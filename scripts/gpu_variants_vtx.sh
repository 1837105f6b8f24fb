# build variants of the per-vertex kernel on the C4 bench (two passes each, inner-stage ms)
for pass in 1 2; do
for f in paper_conf_ipps_adamsbkw22_b200/liblandau.so build_variants/liblandau_*.so; do
  n=$(basename $f .so)
  LANDAU_LIB=$f python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/v_$n.json 2>gpurun_out/v_$n.err
  python -c "import json; d=json.load(open('gpurun_out/v_$n.json')); print('$pass $n', round(d['value']), 'builds/s inner', round(d['stage_ms_per_step']['inner'],3), 'ms')" || tail -3 gpurun_out/v_$n.err
done
done
