# compute-sanitizer over every kernel, the parity report, and one ncu capture of the band LU kernel
{ echo "# compute-sanitizer on scripts/sanitize_run.py (C1, C3 CSR+COO+mass+point_coeffs; C4 16-vertex batch on the symmetric, mirror-slot and per-vertex kernels; pipelined host entry; band LU + solve + implicit step), one B200, round 1"
for t in memcheck racecheck initcheck; do echo "## $t"; timeout 900 compute-sanitizer --tool $t python scripts/sanitize_run.py 2>&1 | grep -E "stats|^ok|SUMMARY|Error|error" | head -20; done; } > gpurun_out/sanitizers.txt 2>&1
tail -3 gpurun_out/sanitizers.txt
python tools/parity_report.py > gpurun_out/parity.json 2>gpurun_out/parity.err; tail -3 gpurun_out/parity.err
bash scripts/gpu_band_ncu.sh
