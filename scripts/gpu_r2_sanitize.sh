# round 2: compute-sanitizer memcheck / racecheck / initcheck / synccheck over scripts/sanitize_run.py
# (default kernels) and its "tail" mode (the fused N3+N4 kernel), plus the parity-margin report
{ echo "# compute-sanitizer on scripts/sanitize_run.py, one B200, round 2 (see the script's header for the kernels covered)"
for mode in default tail; do for t in memcheck racecheck initcheck synccheck; do echo "## $mode $t"; timeout 1200 compute-sanitizer --tool $t python scripts/sanitize_run.py $mode 2>&1 | grep -E "stats|^ok|SUMMARY|Error|error|Hazard|hazard" | head -20; done; done; } > gpurun_out/r02_sanitizers.txt 2>&1
timeout 900 python tools/parity_report.py > gpurun_out/r02_parity_margins.json 2> gpurun_out/r02_parity_margins.err
