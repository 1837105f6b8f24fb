for f in paper_conf_ipps_adamsbkw22_b200/liblandau.so build_variants/liblandau_sf8.so build_variants/liblandau_sf2.so; do for B in 16 64; do
LANDAU_LIB=$f LANDAU_SF_BLOCKS_PER_SM=$B python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bs.json 2>gpurun_out/bs.err
python -c "import json; d=json.load(open('gpurun_out/bs.json')); print('$(basename $f) bps $B', round(d['value']), round(d['stage_ms_per_step']['element'],4))" || tail -3 gpurun_out/bs.err
done; done
