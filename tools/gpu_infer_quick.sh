mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_infer.py -m gpu -x -q -p no:cacheprovider 2>&1 | tail -5 > gpurun_out/pytest_infer.txt
for cfg in "64 2" "32 2" "32 3" "16 3"; do set -- $cfg; SNN_INFER_RING=$1 SNN_INFER_MINB=$2 timeout 300 python tools/bench_infer.py > gpurun_out/bench_infer_r$1_mb$2.json 2>> gpurun_out/bench_infer.err; done
cat gpurun_out/pytest_infer.txt; for f in gpurun_out/bench_infer_r*.json; do python -c "import json,sys; d=json.load(open('$f')); print('$f', d['value'], d['ms_per_call'])"; done; tail -3 gpurun_out/bench_infer.err
