# round 2, after the 3D Jacobian and the column-warp band kernel: compute-sanitizer over
# scripts/sanitize_run.py (default kernels incl. the 3D Jacobian) and its "bandcw" mode
{ echo "# compute-sanitizer on scripts/sanitize_run.py, one B200, round 2 final (see the script's header for the kernels covered)"
for mode in default bandcw; do for t in memcheck racecheck initcheck synccheck; do echo "## $mode $t"; timeout 1500 compute-sanitizer --tool $t python scripts/sanitize_run.py $mode 2>&1 | grep -E "stats|^ok|SUMMARY|Error|error|Hazard|hazard" | head -20; done; done; } > gpurun_out/r02_sanitizers2.txt 2>&1
