{ echo "# compute-sanitizer on scripts/sanitize_run.py (C1, C3 single builds: mirror-directed kernel, CSR+COO+mass+point_coeffs; C4 16-vertex batch on the symmetric, mirror-slot and per-vertex kernels; pipelined host entry; band LU + solve + implicit step; 3D Cartesian inner integral; an emulated pair-split rank), one B200, round 1"
for t in memcheck racecheck initcheck; do echo "## $t"; timeout 900 compute-sanitizer --tool $t python scripts/sanitize_run.py 2>&1 | grep -E "stats|^ok|SUMMARY|Error|error" | head -20; done; } > gpurun_out/sanitizers.txt 2>&1
cat gpurun_out/sanitizers.txt
