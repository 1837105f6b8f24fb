python -m pytest tests/ -x -q -m gpu 2>&1 | tail -2
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
for W in C1 C2 C3; do for MD in 1 0; do
LANDAU_MDIR=$MD python bench.py --workload $W --steps 20 --warmup 5 --no-cpu-baseline > gpurun_out/bm.json 2>gpurun_out/bm.err
python -c "import json; d=json.load(open('gpurun_out/bm.json')); print('$W mdir $MD', round(d['value']), round(d['ms_per_step']*1e3,1), 'us', {k: round(v*1e3,1) for k,v in d['stage_ms_per_step'].items() if v}, d['roofline']['inner_path'])" || tail -3 gpurun_out/bm.err
done; done
M=sm__sass_thread_inst_executed_op_dfma_pred_on.sum,sm__sass_thread_inst_executed_op_dmul_pred_on.sum,sm__sass_thread_inst_executed_op_dadd_pred_on.sum,gpu__time_duration.sum,sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active
ncu --metrics $M --clock-control none -k regex:inner_mdir_kernel -s 2 -c 1 --csv python bench.py --workload C2 --steps 1 --warmup 1 --no-cpu-baseline 2>/dev/null | grep -E '"(sm__|gpu__)' > gpurun_out/flops_mdir.csv
awk -F'","' '{print $(NF-2), $NF}' gpurun_out/flops_mdir.csv
