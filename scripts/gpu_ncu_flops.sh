# FP64 op counts of the inner kernels on the C4 workload (for bench.py's FLOP-per-evaluation constants)
M=sm__sass_thread_inst_executed_op_dfma_pred_on.sum,sm__sass_thread_inst_executed_op_dmul_pred_on.sum,sm__sass_thread_inst_executed_op_dadd_pred_on.sum,gpu__time_duration.sum,sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active
ncu --metrics $M --clock-control none -k regex:inner_vtx_kernel -s 1 -c 1 --csv python bench.py --steps 1 --warmup 1 --no-cpu-baseline 2>/dev/null | grep -E '"(sm__|gpu__)' > gpurun_out/flops_vtx.csv
LANDAU_VTX_MIN_BATCH_PER_SM=100000 ncu --metrics $M --clock-control none -k regex:inner_mir_kernel -s 1 -c 1 --csv python bench.py --steps 1 --warmup 1 --no-cpu-baseline 2>/dev/null | grep -E '"(sm__|gpu__)' > gpurun_out/flops_mir.csv
LANDAU_MIRROR=0 ncu --metrics $M --clock-control none -k regex:inner_sym_kernel -s 1 -c 1 --csv python bench.py --steps 1 --warmup 1 --no-cpu-baseline 2>/dev/null | grep -E '"(sm__|gpu__)' > gpurun_out/flops_sym.csv
LANDAU_SYM=0 LANDAU_MDIR=0 ncu --metrics $M --clock-control none -k regex:"inner_kernel" -s 1 -c 1 --csv python bench.py --steps 1 --warmup 1 --no-cpu-baseline 2>/dev/null | grep -E '"(sm__|gpu__)' > gpurun_out/flops_dir.csv
LANDAU_SYM=0 ncu --metrics $M --clock-control none -k regex:"inner_mdir_kernel" -s 1 -c 1 --csv python bench.py --steps 1 --warmup 1 --no-cpu-baseline 2>/dev/null | grep -E '"(sm__|gpu__)' > gpurun_out/flops_mdir.csv
ncu --metrics $M --clock-control none -k regex:"inner3d_kernel" -s 1 -c 1 --csv python bench.py --steps 1 --warmup 1 --no-cpu-baseline 2>/dev/null | grep -E '"(sm__|gpu__)' > gpurun_out/flops_3d.csv
for f in vtx mir sym dir mdir 3d; do echo "== $f"; awk -F'","' '{print $(NF-2), $NF}' gpurun_out/flops_$f.csv; done
