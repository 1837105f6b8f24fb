# inner-kernel variants on the C4 bench (and C2 single build)
for V in ${VARIANTS:-0 1 2 4}; do
  LANDAU_INNER_VARIANT=$V python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bench_v$V.json 2> gpurun_out/bench_v$V.err
  python -c "import json; d=json.load(open('gpurun_out/bench_v$V.json')); print('V=$V', round(d['value']), 'builds/s inner', round(d['stage_ms_per_step']['inner'],3), 'ms step', round(d['ms_per_step'],3))" || tail -5 gpurun_out/bench_v$V.err
done
