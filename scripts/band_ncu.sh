timeout 300 python scripts/band_only.py > gpurun_out/band_only.log 2>&1
LANDAU_BAND_CW=0 timeout 300 python scripts/band_only.py >> gpurun_out/band_only.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:band_lu_cw -s 1 -c 1 -o gpurun_out/band_cw python scripts/band_only.py > gpurun_out/band_cw_ncu.log 2>&1
