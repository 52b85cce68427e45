mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_sharding.py tests/test_gpu_parity.py -m gpu -q -p no:cacheprovider -x -k "shard or C1 or C4 or batch" 2>&1 | tail -5 > gpurun_out/pytest_gpu.txt
timeout 600 python bench.py --no-infer --cpu-images 0 > gpurun_out/bench.json 2> gpurun_out/bench.err
timeout 300 python bench.py --no-infer --cpu-images 0 --local-shards 2 --no-floor > gpurun_out/bench_ls2.json 2>> gpurun_out/bench.err
cat gpurun_out/pytest_gpu.txt
python -c "
import json
for f in ('bench','bench_ls2'):
    d=json.load(open('gpurun_out/%s.json'%f)); print(f, d['value'], d['config']['parallelism'])
"; tail -3 gpurun_out/bench.err
