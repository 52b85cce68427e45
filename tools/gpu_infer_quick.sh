mkdir -p gpurun_out
SNN_INFER_RING=40 timeout 240 python -m pytest tests/test_gpu_infer.py -m gpu -x -q -p no:cacheprovider 2>&1 | tail -3 > gpurun_out/pytest_infer.txt
timeout 240 python -m pytest tests/test_gpu_infer.py -m gpu -x -q -p no:cacheprovider 2>&1 | tail -3 >> gpurun_out/pytest_infer.txt
cat gpurun_out/pytest_infer.txt
for r in 32 40; do SNN_INFER_RING=$r timeout 120 python tools/bench_infer.py > gpurun_out/bi_$r.json 2>> gpurun_out/bench_infer.err; python -c "import json; d=json.load(open('gpurun_out/bi_$r.json')); print('$r', d['value'])"; done
tail -2 gpurun_out/bench_infer.err
