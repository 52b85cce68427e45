# quick iteration: lean-kernel parity subset + bench + epoch trace
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -p no:cacheprovider -x -k "C1 or C4 or batch or ragged or stepwise or cluster or zero or raster or C2_C3" 2>&1 | tail -4 > gpurun_out/pytest_gpu.txt
timeout 600 python bench.py --no-infer --cpu-images 0 > gpurun_out/bench.json 2> gpurun_out/bench.err
timeout 120 python tools/trace_lean.py --images 8 > gpurun_out/trace_lean.txt 2>&1
cat gpurun_out/pytest_gpu.txt | cut -c1-200
python -c "
import json
d=json.load(open('gpurun_out/bench.json')); print('bench', d['value'], d['e2e']['value'], 'epochs', d['secondary']['epochs_per_image'], 'resim', d['secondary']['resims_per_image'], 'hz', d['secondary']['log_stops_per_image'], d['clocks']['sm_mhz'], d['clocks']['reasons'])
"; tail -2 gpurun_out/bench.err; cat gpurun_out/trace_lean.txt
SNN_LIB_PATH=exp_libs/libsnn_cyc.so timeout 120 python tools/trace_lean.py --images 8 > gpurun_out/trace_lean_cyc.txt 2>&1; grep "cycles/epoch\|warp-steps" gpurun_out/trace_lean_cyc.txt
