# per-vertex mirror kernel: parity, then C4 bench (auto = per-vertex) vs the slot kernel at several batch sizes
python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "vertex or symmetric or coincident" 2>&1 | tail -3
for B in 1024 512 256 128; do
  for V in 3 100000; do
    LANDAU_VTX_MIN_BATCH_PER_SM=$V python bench.py --batch $B --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bench_vtx_${B}_$V.json 2> gpurun_out/bench_vtx_${B}_$V.err
    python -c "import json; d=json.load(open('gpurun_out/bench_vtx_${B}_$V.json')); print('B=$B V=$V', round(d['value']), 'builds/s', round(d['ms_per_step'],3), 'ms', {k: round(v,3) for k,v in d['stage_ms_per_step'].items() if v}, 'frac', round(d['roofline']['frac'],3), d['roofline']['inner_path'])" || tail -5 gpurun_out/bench_vtx_${B}_$V.err
  done
done
