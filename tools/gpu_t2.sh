mkdir -p gpurun_out
timeout 300 python -m pytest tests/test_gpu_16bit.py -x -q -p no:cacheprovider 2>&1 | tail -5 > gpurun_out/pytest_16.txt
timeout 300 python tools/bench_table2.py > gpurun_out/bench_table2.json 2> gpurun_out/bench_table2.err
cat gpurun_out/pytest_16.txt; cut -c1-400 gpurun_out/bench_table2.json; tail -3 gpurun_out/bench_table2.err
