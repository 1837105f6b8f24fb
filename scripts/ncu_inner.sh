# ncu --set full of the per-vertex inner kernel on the C4 bench (1 GPU), source-level stalls
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"inner_vtx_kernel" -s 1 -c 1 \
  -o gpurun_out/r2_inner python bench.py --steps 1 --warmup 1 --no-sublines --no-cpu-baseline > gpurun_out/r2_inner_ncu.log 2>&1
echo "ncu rc=$?" >> gpurun_out/r2_inner_ncu.log
