# A/B of the current library against exp_libs/libsnn_old.so on one box (bench value), after the lean parity tests
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_sharding.py -m gpu -q -p no:cacheprovider -x 2>&1 | tail -2
for lib in new old new old; do
  if [ $lib = old ]; then export SNN_LIB_PATH=exp_libs/libsnn_old.so; else unset SNN_LIB_PATH; fi
  timeout 600 python bench.py --no-infer --cpu-images 0 --no-floor > gpurun_out/ab_$lib.json 2>/dev/null
  python -c "
import json
d=json.load(open('gpurun_out/ab_$lib.json')); e=d['secondary'].get('epochs_per_image'); v=d['value']; print('$lib', round(v,1), 'epochs', e, 'us/epoch', round(1e6/v/e,3))
"
done
