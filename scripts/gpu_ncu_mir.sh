# one ncu --set full capture of the mirror inner kernel (C4) for the source/stall view
M=sm__sass_thread_inst_executed_op_dfma_pred_on.sum,sm__sass_thread_inst_executed_op_dmul_pred_on.sum,sm__sass_thread_inst_executed_op_dadd_pred_on.sum,sm__sass_thread_inst_executed_op_fp64_pred_on.sum
ncu --set full --metrics $M --clock-control none --import-source on -k regex:inner_mir_kernel -s 1 -c 1 -o gpurun_out/mir_full python bench.py --steps 1 --warmup 1 --no-cpu-baseline > gpurun_out/ncu_mir.log 2>&1
tail -1 gpurun_out/ncu_mir.log
