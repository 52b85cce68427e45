# layout sweep of the event engine on C4 (bench.py, no cpu baseline)
for ls in 1 2 4 8; do for cs in 8 16; do for cpt in 1 2 4; do
  SNN_CPT=$cpt timeout 200 python bench.py --steps 5 --warmup 3 --cpu-images 0 --images-per-step 16 --local-shards $ls --cluster-size $cs 2>&1 | tail -1 | python -c "
import json,sys
s=sys.stdin.read()
try:
  d=json.loads(s); print('ls=$ls cs=$cs cpt=$cpt', d['config']['cluster_size'], d['config']['threads_per_cta'], round(d['value'],1), 'img/s epochs/img', round(d['secondary']['epochs_per_image'],2))
except Exception: print('ls=$ls cs=$cs cpt=$cpt FAILED', s[-200:])
"
done; done; done
