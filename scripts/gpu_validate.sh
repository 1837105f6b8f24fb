# Re-entry validation: GPU tests, smoke(), default bench line.
python -m pytest tests/ -q -m gpu > gpurun_out/pytest_gpu.log 2>&1; tail -3 gpurun_out/pytest_gpu.log
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -2
python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err; cat gpurun_out/bench_default.json
python scripts/band_timing.py > gpurun_out/band_timing.txt 2>&1; tail -5 gpurun_out/band_timing.txt
