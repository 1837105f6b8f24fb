M=sm__sass_thread_inst_executed_op_dfma_pred_on.sum,sm__sass_thread_inst_executed_op_dmul_pred_on.sum,sm__sass_thread_inst_executed_op_dadd_pred_on.sum,sm__sass_thread_inst_executed_op_fp64_pred_on.sum
ncu --set full --metrics $M --clock-control none --import-source on -k regex:inner_sym_kernel -s 1 -c 1 -o gpurun_out/inner_sym python bench.py --steps 1 --warmup 1 --no-cpu-baseline > gpurun_out/ncu_sym.log 2>&1
tail -1 gpurun_out/ncu_sym.log
ncu --metrics gpu__time_duration.sum --clock-control none -c 200 --csv --log-file gpurun_out/launches_sym.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline > /dev/null 2>&1
