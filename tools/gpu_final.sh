mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi.txt
timeout 900 python -m pytest tests -m gpu -q -p no:cacheprovider 2>&1 | tail -6 > gpurun_out/pytest_gpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.txt 2>&1
timeout 600 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err
timeout 300 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/bench_ref.json 2>> gpurun_out/bench.err
timeout 200 python tools/bench_ensemble.py --nets 64 --images 8 > gpurun_out/bench_ensemble64.json 2>> gpurun_out/bench.err
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 3 --images-per-step 8 --cpu-images 0 --no-infer > gpurun_out/bench_ncu.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:present_ --launch-skip 1 -c 1 -o gpurun_out/full -f python tools/ncu_target.py --images 32 > gpurun_out/ncu_full.log 2>&1
python tools/ncu_summary.py gpurun_out/full.ncu-rep gpurun_out/ncu_full_latest.json --images 32 --source "r01 final: ncu --set full -k regex:present_ --launch-skip 1 -c 1 tools/ncu_target.py --images 32" > /dev/null 2>&1
cat gpurun_out/pytest_gpu.txt gpurun_out/smoke.txt | cut -c1-150
python -c "
import json
d=json.load(open('gpurun_out/bench.json')); print('bench', d['value'], d['e2e']['value'], d['roofline']['frac'], d['roofline']['traffic'], d['inference']['value'], d['clocks'])
print('ref', open('gpurun_out/bench_ref.json').read()[:200])
print('ens64', open('gpurun_out/bench_ensemble64.json').read()[:250])
"; tail -3 gpurun_out/bench.err
