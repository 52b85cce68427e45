mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi.txt
timeout 600 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err
timeout 300 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29512 bench.py --gpus 2 --steps 3 --images-per-step 8 --infer-images 512 > gpurun_out/bench_2rank.json 2>> gpurun_out/bench.err
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 3 --images-per-step 8 --cpu-images 0 --no-infer > gpurun_out/bench_ncu.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:present_ --launch-skip 1 -c 1 -o gpurun_out/full -f python tools/ncu_target.py --images 32 > gpurun_out/ncu_full.log 2>&1
python tools/ncu_summary.py gpurun_out/full.ncu-rep gpurun_out/ncu_full_latest.json --images 32 --source "r01 final: ncu --set full -k regex:present_ --launch-skip 1 -c 1 tools/ncu_target.py --images 32" > /dev/null 2>&1
timeout 300 ncu --set full --clock-control none --import-source on -k infer_kernel -c 1 -o gpurun_out/infer_full -f python tools/bench_infer.py --images 1332 --steps 1 --warmup 1 > gpurun_out/ncu_infer.log 2>&1
python tools/ncu_summary.py gpurun_out/infer_full.ncu-rep gpurun_out/ncu_infer_latest.json --images 1332 --source "r01 final: ncu --set full -k infer_kernel -c 1 tools/bench_infer.py --images 1332" > /dev/null 2>&1
python -c "
import json
d=json.load(open('gpurun_out/bench.json')); print('N1', d['value'], d['e2e']['value'], d['roofline']['frac'], d['roofline']['traffic'], d['inference']['value'])
for l in open('gpurun_out/bench_2rank.json'):
    if l.startswith('{'): d=json.loads(l); print('N2', d['value'], d['config']['parallelism'], (d.get('inference') or {}).get('value'))
"; tail -3 gpurun_out/bench.err; grep dram_bytes gpurun_out/ncu_full_latest.json gpurun_out/ncu_infer_latest.json
