mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_sparse.py -x -q -p no:cacheprovider 2>&1 | tail -40 > gpurun_out/pytest_sparse.txt
timeout 300 python tools/bench_sparse.py > gpurun_out/bench_sparse.json 2> gpurun_out/bench_sparse.err
tail -3 gpurun_out/pytest_sparse.txt; cat gpurun_out/bench_sparse.json; tail -3 gpurun_out/bench_sparse.err
