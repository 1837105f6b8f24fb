# round 2 evidence: default bench line, ncu launch list of the same command, ncu --set full of the
# headline inner kernel, and the C2-ncu single-build inner kernel (fused and stand-alone)
set -x
timeout 900 python bench.py > gpurun_out/r02_bench_default.json 2> gpurun_out/r02_bench_default.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 600 --csv --log-file gpurun_out/r02_launches.csv \
  python bench.py --steps 2 --warmup 1 --no-sublines --no-cpu-baseline > /dev/null 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"inner_vtx_kernel|element_sf_kernel|assemble_kernel|field_kernel" -s 4 -c 4 \
  -o gpurun_out/r02_c4_full python bench.py --steps 1 --warmup 1 --no-sublines --no-cpu-baseline > gpurun_out/r02_c4_full.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"single_build_kernel" -s 3 -c 1 \
  -o gpurun_out/r02_c2ncu_fused python bench.py --workload C2ncu --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/r02_c2ncu_fused.log 2>&1
LANDAU_FUSED_SINGLE=0 timeout 600 ncu --set full --clock-control none --import-source on -k regex:"inner_mdir_kernel" -s 3 -c 1 \
  -o gpurun_out/r02_c2ncu_mdir python bench.py --workload C2ncu --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/r02_c2ncu_mdir.log 2>&1
timeout 300 python bench.py --workload C2ncu --no-cpu-baseline > gpurun_out/r02_bench_C2ncu.json 2>/dev/null
for W in C1 C2 C3 C5; do timeout 600 python bench.py --workload $W > gpurun_out/r02_bench_$W.json 2>/dev/null; done
timeout 300 python bench.py --batch 128 --no-sublines --no-cpu-baseline > gpurun_out/r02_bench_b128.json 2>/dev/null
