mkdir -p gpurun_out
for mb in 3 4; do SNN_INFER_MINB=$mb timeout 120 python tools/bench_infer.py > gpurun_out/bench_infer_mb$mb.json 2>> gpurun_out/bench_infer.err; done
for mb in 3 4; do python -c "import json; d=json.load(open('gpurun_out/bench_infer_mb$mb.json')); print($mb, d['value'])"; done; tail -3 gpurun_out/bench_infer.err
