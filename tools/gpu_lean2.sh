mkdir -p gpurun_out
timeout 300 python -m pytest tests/test_gpu_parity.py tests/test_gpu_sharding.py -m gpu -x -q -p no:cacheprovider 2>&1 | tail -15 > gpurun_out/pytest_lean2.txt
timeout 60 python tools/trace_lean.py --images 8 > gpurun_out/trace_lean.txt 2>&1
timeout 120 python bench.py --steps 10 --cpu-images 0 --no-infer > gpurun_out/bench_quick.json 2>/dev/null
tail -3 gpurun_out/pytest_lean2.txt; cat gpurun_out/trace_lean.txt; python -c "import json; d=json.load(open('gpurun_out/bench_quick.json')); print(d['value'], d['secondary']['epochs_per_image'], d['secondary']['log_stops_per_image'])"
