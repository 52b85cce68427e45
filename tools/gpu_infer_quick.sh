mkdir -p gpurun_out
timeout 240 python -m pytest tests/test_gpu_infer.py -m gpu -x -q -p no:cacheprovider 2>&1 | tail -5 > gpurun_out/pytest_infer.txt
timeout 120 python tools/bench_infer.py > gpurun_out/bench_infer.json 2> gpurun_out/bench_infer.err
tail -3 gpurun_out/pytest_infer.txt; python -c "import json; d=json.load(open('gpurun_out/bench_infer.json')); print(d['value'])"; tail -3 gpurun_out/bench_infer.err
