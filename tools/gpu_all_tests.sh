mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q -p no:cacheprovider 2>&1 | tail -8 > gpurun_out/pytest_gpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.txt 2>&1
timeout 900 python tools/bench_schedule.py > gpurun_out/bench_schedule.jsonl 2> gpurun_out/bench_schedule.err
cat gpurun_out/pytest_gpu.txt gpurun_out/smoke.txt; python -c "
import json
for l in open('gpurun_out/bench_schedule.jsonl'):
    d=json.loads(l); print(d['schedule'], round(d['train_images_per_s'],1), d['final_error'], [(p['images'], round(p['sim_s'],1), round(p['device_s'],3), round(p['error'],3)) for p in d['curve']])
"; tail -3 gpurun_out/bench_schedule.err
