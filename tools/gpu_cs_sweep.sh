mkdir -p gpurun_out
for cs in 16 15 14 13 12 16; do
  timeout 600 python bench.py --no-infer --cpu-images 0 --no-floor --cluster-size $cs > gpurun_out/cs_$cs.json 2>/dev/null
  python -c "
import json
d=json.load(open('gpurun_out/cs_$cs.json')); e=d['secondary'].get('epochs_per_image'); v=d['value']; print('cs $cs', round(v,1), 'epochs', e, 'us/epoch', round(1e6/v/e,3))
"
done
