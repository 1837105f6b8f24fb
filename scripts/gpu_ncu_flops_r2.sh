# FP64 op counts of the inner kernels on the C4 workload (bench.py's FLOP-per-evaluation constants),
# with the bench line of each run (its flops_per_launch / flop_per_pair = the evaluations per launch)
M=sm__sass_thread_inst_executed_op_dfma_pred_on.sum,sm__sass_thread_inst_executed_op_dmul_pred_on.sum,sm__sass_thread_inst_executed_op_dadd_pred_on.sum,gpu__time_duration.sum
run() {   # name, kernel regex, env...
  name=$1; k=$2; shift 2
  env "$@" ncu --metrics $M --clock-control none -k regex:$k -s 1 -c 1 --csv --log-file gpurun_out/flops2_$name.csv python bench.py --steps 1 --warmup 1 --no-sublines --no-cpu-baseline > gpurun_out/flops2_$name.json 2>/dev/null
}
run vtx inner_vtx_kernel X=1
run mir inner_mir_kernel LANDAU_VTX_MIN_WEIGHT_PER_SM=100000000
run sym inner_sym_kernel LANDAU_MIRROR=0
run dir "inner_kernel" LANDAU_SYM=0 LANDAU_MDIR=0 LANDAU_VTX_MIN_WEIGHT_PER_SM=100000000
run mdir inner_mdir_kernel LANDAU_SYM=0 LANDAU_VTX_MIN_WEIGHT_PER_SM=100000000
