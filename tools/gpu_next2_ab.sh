# NEXT-2 throughput A/B: the current library against exp_libs/libsnn_old.so on one box
mkdir -p gpurun_out
for lib in new old; do
  if [ $lib = old ]; then export SNN_LIB_PATH=exp_libs/libsnn_old.so; else unset SNN_LIB_PATH; fi
  timeout 600 python tools/bench_next2.py --no-oracle > gpurun_out/n2_$lib.jsonl 2>/dev/null
  python -c "
import json
for l in open('gpurun_out/n2_$lib.jsonl'):
    d=json.loads(l); print('$lib', d['config'], round(d['images_per_s'],1), round(d['us_per_step'],3))
"
done
