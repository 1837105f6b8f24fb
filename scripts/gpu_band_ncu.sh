# band LU: launch durations and one full ncu capture of the factor kernel
ncu --metrics gpu__time_duration.sum --clock-control none -k regex:band --csv --log-file gpurun_out/band_launches.csv python scripts/band_timing.py 64 > /dev/null 2>&1
python tools/ncu_launches.py gpurun_out/band_launches.csv 2>/dev/null | head -20 || tail -20 gpurun_out/band_launches.csv
ncu --set full --clock-control none --import-source on -k regex:band_lu -s 2 -c 1 -o gpurun_out/band_full python scripts/band_timing.py 1024 > gpurun_out/band_ncu.log 2>&1
tail -3 gpurun_out/band_ncu.log
