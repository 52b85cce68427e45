mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi.txt
timeout 600 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err
timeout 300 python bench.py --local-shards 2 --steps 5 --cpu-images 0 --no-infer > gpurun_out/bench_ls2.json 2>> gpurun_out/bench.err
timeout 300 python bench.py --local-shards 4 --steps 5 --cpu-images 0 --no-infer > gpurun_out/bench_ls4.json 2>> gpurun_out/bench.err
timeout 300 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29511 bench.py --gpus 2 --mode shard --steps 3 --images-per-step 8 > gpurun_out/bench_shard2_shared_gpu.json 2>> gpurun_out/bench.err
timeout 300 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/bench_ref.json 2>> gpurun_out/bench.err
for f in bench bench_ls2 bench_ls4 bench_shard2_shared_gpu bench_ref; do echo "== $f"; python -c "
import json
for l in open('gpurun_out/$f.json'):
    l=l.strip()
    if l.startswith('{'):
        d=json.loads(l); print(d.get('value'), d.get('unit'), d.get('config',{}).get('parallelism'), (d.get('inference') or {}).get('value'), (d.get('inference') or {}).get('roofline',{}).get('frac'))
"; done
tail -5 gpurun_out/bench.err
