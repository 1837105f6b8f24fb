# per-vertex mirror kernel: variants on the C4 bench, then one ncu --set full capture (FLOP counts, stalls)
for f in paper_conf_ipps_adamsbkw22_b200/liblandau.so build_variants/liblandau_*.so; do
  n=$(basename $f .so)
  LANDAU_LIB=$f python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/v_$n.json 2>gpurun_out/v_$n.err
  python -c "import json; d=json.load(open('gpurun_out/v_$n.json')); print('$n', round(d['value']), 'builds/s inner', round(d['stage_ms_per_step']['inner'],3), 'ms')" || tail -3 gpurun_out/v_$n.err
done
M=sm__sass_thread_inst_executed_op_dfma_pred_on.sum,sm__sass_thread_inst_executed_op_dmul_pred_on.sum,sm__sass_thread_inst_executed_op_dadd_pred_on.sum,sm__sass_thread_inst_executed_op_fp64_pred_on.sum
ncu --set full --metrics $M --clock-control none --import-source on -k regex:inner_vtx_kernel -s 1 -c 1 -o gpurun_out/vtx_full python bench.py --steps 1 --warmup 1 --no-cpu-baseline > gpurun_out/ncu_vtx.log 2>&1
tail -1 gpurun_out/ncu_vtx.log
