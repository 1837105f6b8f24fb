M=sm__sass_thread_inst_executed_op_dfma_pred_on.sum,sm__sass_thread_inst_executed_op_dmul_pred_on.sum,sm__sass_thread_inst_executed_op_dadd_pred_on.sum,gpu__time_duration.sum,sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active
LANDAU_SYM=0 LANDAU_MDIR=0 ncu --metrics $M --clock-control none -k regex:"inner_kernel" -s 1 -c 1 --csv python bench.py --steps 1 --warmup 1 --no-cpu-baseline 2>/dev/null | grep -E '"(sm__|gpu__)' > gpurun_out/flops_dir.csv
LANDAU_SYM=0 ncu --metrics $M --clock-control none -k regex:"inner_mdir_kernel" -s 1 -c 1 --csv python bench.py --steps 1 --warmup 1 --no-cpu-baseline 2>/dev/null | grep -E '"(sm__|gpu__)' > gpurun_out/flops_mdir.csv
for f in dir mdir; do echo "== $f"; awk -F'","' '{print $(NF-2), $NF}' gpurun_out/flops_$f.csv; done
