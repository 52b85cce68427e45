# lean-kernel iteration: parity (lean subset + fuzz), bench, epoch trace
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -p no:cacheprovider -x 2>&1 | tail -4 > gpurun_out/pytest_gpu.txt
timeout 600 python bench.py --no-infer --cpu-images 0 > gpurun_out/bench.json 2> gpurun_out/bench.err
timeout 120 python tools/trace_lean.py --images 8 > gpurun_out/trace_lean.txt 2>&1
cat gpurun_out/pytest_gpu.txt | cut -c1-300
python -c "
import json
d=json.load(open('gpurun_out/bench.json')); print('bench', d['value'], d['e2e']['value'], 'epochs', d['secondary'].get('epochs_per_image'), d['clocks']['sm_mhz'], d['clocks']['reasons'], 'floor', d.get('latency_roofline',{}).get('frac'))
"; tail -2 gpurun_out/bench.err; cat gpurun_out/trace_lean.txt
