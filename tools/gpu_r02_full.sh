# r02 full pass: -m gpu suite, smoke, bench (all fields), reference arm, launch list
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi.txt
lscpu > gpurun_out/lscpu.txt 2>&1
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider 2>&1 | tail -15 > gpurun_out/pytest_gpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.txt 2>&1
timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err
timeout 300 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/bench_ref.json 2>> gpurun_out/bench.err
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 3 --cpu-images 0 --no-infer --no-floor > gpurun_out/bench_ncu.log 2>&1
cat gpurun_out/pytest_gpu.txt | cut -c1-200; cat gpurun_out/smoke.txt | tail -2
python - <<'PY'
import json
d=json.load(open('gpurun_out/bench.json'))
print('bench', d['value'], 'e2e', d['e2e']['value'], 'clocks', d['clocks'])
print('roofline', {k: d['roofline'][k] for k in ('achieved','peak','frac','kernel_ms_per_launch','kernel_share_of_step','alg_bytes_per_launch')})
print('floor', d['latency_roofline'])
print('infer', d['inference']['value'], d['inference']['roofline']['frac'], d['inference']['roofline'].get('lif_column_steps_per_image'))
print('cpu', json.dumps(d.get('cpu_baseline'))[:900])
PY
tail -3 gpurun_out/bench.err; head -c 300 gpurun_out/bench_ref.json
