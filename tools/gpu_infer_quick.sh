mkdir -p gpurun_out
timeout 240 python -m pytest tests/test_gpu_infer.py tests/test_gpu_schedule.py -m gpu -x -q -p no:cacheprovider 2>&1 | tail -4 > gpurun_out/pytest_infer.txt
cat gpurun_out/pytest_infer.txt
timeout 120 python tools/bench_infer.py > gpurun_out/bi.json 2>> gpurun_out/bench_infer.err; python -c "import json; d=json.load(open('gpurun_out/bi.json')); print(d['value'], d['post_spikes_per_image'])"
tail -2 gpurun_out/bench_infer.err
