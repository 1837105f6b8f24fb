# round 2: GPU tests then the default bench line (all sub-lines)
timeout 900 python -m pytest tests/ -x -q -m gpu > gpurun_out/r2_tests.log 2>&1
echo "tests rc=$?" >> gpurun_out/r2_tests.log
timeout 900 python bench.py > gpurun_out/r2_bench.json 2> gpurun_out/r2_bench.err
echo "bench rc=$?" >> gpurun_out/r2_bench.err
