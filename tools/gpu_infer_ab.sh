# inference A/B: the current library against exp_libs/libsnn_old.so (same box), plus the inference parity tests
mkdir -p gpurun_out
timeout 400 python -m pytest tests/test_gpu_infer.py -m gpu -x -q -p no:cacheprovider 2>&1 | tail -3
for lib in new old new old; do
  if [ $lib = old ]; then export SNN_LIB_PATH=exp_libs/libsnn_old.so; else unset SNN_LIB_PATH; fi
  timeout 120 python tools/bench_infer.py > gpurun_out/bi_$lib.json 2>/dev/null
  python -c "import json; d=json.load(open('gpurun_out/bi_$lib.json')); print('$lib', round(d['value']), d['post_spikes_per_image'])"
done
