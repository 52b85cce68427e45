# final check at HEAD: the whole -m gpu suite, smoke, one bench line
mkdir -p gpurun_out/check
timeout 1500 python -m pytest tests -m gpu -q -rs -p no:cacheprovider 2>&1 | tail -6 > gpurun_out/check/pytest_gpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/check/smoke.txt 2>&1
timeout 900 python bench.py > gpurun_out/check/bench.json 2> gpurun_out/check/bench.err
cat gpurun_out/check/pytest_gpu.txt; tail -1 gpurun_out/check/smoke.txt | cut -c1-120
python -c "
import json; d=json.load(open('gpurun_out/check/bench.json')); print('bench', d['value'], 'e2e', d['e2e']['value'], 'floor', d['latency_roofline']['frac'], 'clocks', d['clocks'], 'launches', d['gpu_launches'])"
