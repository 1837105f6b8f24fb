ncu --set full --clock-control none --import-source on -k regex:band_lu -s 2 -c 1 -o gpurun_out/band_full2 python scripts/band_timing.py 1024 > gpurun_out/band_ncu2.log 2>&1
tail -1 gpurun_out/band_ncu2.log
