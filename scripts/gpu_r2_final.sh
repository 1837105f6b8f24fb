# round 2 final evidence (after the trace correction and the 16-chunk host entry): GPU tests, default
# bench line, ncu launch list of the same command, ncu --set full of the C4 kernels, per-config bench
# lines, the 128-vertex line, the reference arm, the parity margins, compute-sanitizer over every kernel
set -x
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r02f_pytest_gpu.log 2>&1
python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > gpurun_out/r02f_smoke.log 2>&1
timeout 900 python bench.py > gpurun_out/r02f_bench_default.json 2> gpurun_out/r02f_bench_default.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 600 --csv --log-file gpurun_out/r02f_launches.csv \
  python bench.py --steps 2 --warmup 1 --no-sublines --no-cpu-baseline > /dev/null 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"inner_vtx_kernel|element_sf_kernel|assemble_kernel|field_kernel" -s 4 -c 4 \
  -o gpurun_out/r02f_c4_full python bench.py --steps 1 --warmup 1 --no-sublines --no-cpu-baseline > gpurun_out/r02f_c4_full.log 2>&1
for W in C1 C2 C3 C5; do timeout 600 python bench.py --workload $W > gpurun_out/r02f_bench_$W.json 2>/dev/null; done
timeout 300 python bench.py --workload C2ncu --no-cpu-baseline > gpurun_out/r02f_bench_C2ncu.json 2>/dev/null
timeout 300 python bench.py --batch 128 --no-sublines --no-cpu-baseline > gpurun_out/r02f_bench_b128.json 2>/dev/null
timeout 600 python bench.py --impl reference > gpurun_out/r02f_bench_reference.json 2> gpurun_out/r02f_bench_reference.err
timeout 1200 python tools/parity_report.py > gpurun_out/r02f_parity_margins.json 2> gpurun_out/r02f_parity.err
python scripts/band_timing.py > gpurun_out/r02f_band_timing.txt 2>&1
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > gpurun_out/r02f_smi.csv
{ echo "# compute-sanitizer on scripts/sanitize_run.py, one B200, round 2 final code (see the script's header for the kernels covered)"
for t in memcheck racecheck initcheck synccheck; do echo "## default $t"; timeout 1500 compute-sanitizer --tool $t python scripts/sanitize_run.py 2>&1 | grep -E "stats|^ok|SUMMARY|Error|error|Hazard|hazard" | head -20; done; } > gpurun_out/r02f_sanitizers.txt 2>&1
