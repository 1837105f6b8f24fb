# round 2 evidence: GPU tests, default bench line, ncu launch list of the same command, ncu --set full
# of the headline inner kernel and the FE kernels, the C2-ncu single-build inner kernel (slot kernel:
# the automatic path at H = 2176) and the C2 fused single-build kernel, per-config bench lines, the
# 128-vertex line, the reference arm, and the parity margins
set -x
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r02_pytest_gpu.log 2>&1
timeout 900 python bench.py > gpurun_out/r02_bench_default.json 2> gpurun_out/r02_bench_default.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 600 --csv --log-file gpurun_out/r02_launches.csv \
  python bench.py --steps 2 --warmup 1 --no-sublines --no-cpu-baseline > /dev/null 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"inner_vtx_kernel|element_sf_kernel|assemble_kernel|field_kernel" -s 4 -c 4 \
  -o gpurun_out/r02_c4_full python bench.py --steps 1 --warmup 1 --no-sublines --no-cpu-baseline > gpurun_out/r02_c4_full.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"inner_mir_kernel|reduce_mir_kernel" -s 2 -c 2 \
  -o gpurun_out/r02_c2ncu_full python bench.py --workload C2ncu --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/r02_c2ncu_full.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"single_build_kernel" -s 2 -c 1 \
  -o gpurun_out/r02_c2_fused python bench.py --workload C2 --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/r02_c2_fused.log 2>&1
timeout 300 python bench.py --workload C2ncu --no-cpu-baseline > gpurun_out/r02_bench_C2ncu.json 2>/dev/null
for W in C1 C2 C3 C5; do timeout 600 python bench.py --workload $W > gpurun_out/r02_bench_$W.json 2>/dev/null; done
timeout 300 python bench.py --batch 128 --no-sublines --no-cpu-baseline > gpurun_out/r02_bench_b128.json 2>/dev/null
timeout 600 python bench.py --impl reference > gpurun_out/r02_bench_reference.json 2> gpurun_out/r02_bench_reference.err
timeout 1200 python tools/parity_report.py > gpurun_out/r02_parity.json 2> gpurun_out/r02_parity.err
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > gpurun_out/r02_smi.csv
