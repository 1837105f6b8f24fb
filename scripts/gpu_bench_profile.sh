# Round bench + evidence: default bench (with cpu_baseline), small-config lines, the reference arm,
# the ncu launch list of the bench command, FLOP counts and one ncu --set full capture of the dominant
# kernel (inner_vtx_kernel) and of the other kernels.
set -x
python -m pytest tests/ -q -m gpu > gpurun_out/pytest_gpu.log 2>&1; tail -1 gpurun_out/pytest_gpu.log
python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err; cat gpurun_out/bench_default.json
python tools/parity_report.py > gpurun_out/parity.json 2>/dev/null
for w in C1 C2 C3 C5; do python bench.py --workload $w --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bench_$w.json 2>gpurun_out/bench_$w.err; done
python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/bench_reference.json 2> gpurun_out/bench_reference.err; cat gpurun_out/bench_reference.json
ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline > gpurun_out/ncu_launch_bench.log 2>&1
bash scripts/gpu_ncu_flops.sh
M=sm__sass_thread_inst_executed_op_dfma_pred_on.sum,sm__sass_thread_inst_executed_op_dmul_pred_on.sum,sm__sass_thread_inst_executed_op_dadd_pred_on.sum,sm__sass_thread_inst_executed_op_fp64_pred_on.sum
ncu --set full --metrics $M --clock-control none --import-source on -k regex:inner_vtx_kernel -s 1 -c 1 -o gpurun_out/inner_full python bench.py --steps 1 --warmup 1 --no-cpu-baseline > gpurun_out/ncu_full.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:"element_sf_kernel|assemble_kernel|field_kernel" -s 3 -c 3 -o gpurun_out/others_full python bench.py --steps 1 --warmup 1 --no-cpu-baseline > gpurun_out/ncu_others.log 2>&1
tail -2 gpurun_out/ncu_full.log
ncu --set full --clock-control none --import-source on -k regex:band_lu -s 2 -c 1 -o gpurun_out/band_full python scripts/band_timing.py 1024 > gpurun_out/band_ncu.log 2>&1
