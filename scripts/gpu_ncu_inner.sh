# ncu --set full of the inner kernel (C4 workload), both TPT variants, plus FP64 op counts
M=sm__sass_thread_inst_executed_op_dfma_pred_on.sum,sm__sass_thread_inst_executed_op_dmul_pred_on.sum,sm__sass_thread_inst_executed_op_dadd_pred_on.sum,sm__sass_thread_inst_executed_op_fp64_pred_on.sum
for T in ${TPTS:-1 2}; do
LANDAU_INNER_TPT=$T ncu --set full --metrics $M --clock-control none --import-source on -k regex:inner_kernel -s 1 -c 1 -o gpurun_out/inner_t$T python bench.py --steps 1 --warmup 1 --no-cpu-baseline > gpurun_out/ncu_t$T.log 2>&1
tail -2 gpurun_out/ncu_t$T.log
done
