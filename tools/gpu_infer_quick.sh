mkdir -p gpurun_out
for cfg in "32 3" "64 2" "32 2" "16 3"; do set -- $cfg; SNN_INFER_RING=$1 SNN_INFER_MINB=$2 timeout 120 python tools/bench_infer.py > gpurun_out/bi_$1_$2.json 2>> gpurun_out/bench_infer.err; python -c "import json; d=json.load(open('gpurun_out/bi_$1_$2.json')); print('$1 $2', d['value'])"; done
tail -2 gpurun_out/bench_infer.err
