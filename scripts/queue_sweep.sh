for CW in 4 8 12; do for PCT in 25 50 100; do for B in 1024 128; do
LANDAU_VTX_CHUNK_WEIGHT=$CW LANDAU_VTX_CHUNKED_PCT=$PCT timeout 300 python bench.py --batch $B --no-sublines --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('CW$CW PCT$PCT B$B', round(d['ms_per_step'],4), 'inner', round(d['stage_ms_per_step']['inner'],4))"
done; done; done
