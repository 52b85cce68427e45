mkdir -p gpurun_out
timeout 300 python -m pytest tests/test_gpu_schedule.py -x -q -p no:cacheprovider 2>&1 | tail -5 > gpurun_out/pytest_schedule.txt
timeout 900 python tools/bench_schedule.py > gpurun_out/bench_schedule.jsonl 2> gpurun_out/bench_schedule.err
cat gpurun_out/pytest_schedule.txt; python -c "
import json
for l in open('gpurun_out/bench_schedule.jsonl'):
    d=json.loads(l); print(d['schedule'], round(d['train_images_per_s'],1), d['final_error'], [(p['images'], round(p['sim_s'],1), round(p['error'],3)) for p in d['curve']])
"; tail -3 gpurun_out/bench_schedule.err
