# deferred-column lean kernel: parity + bench + step-kernel racecheck recheck
mkdir -p gpurun_out/san
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_sharding.py -m gpu -q -p no:cacheprovider -x 2>&1 | tail -15 > gpurun_out/pytest_gpu.txt
timeout 600 python bench.py --no-infer --cpu-images 0 > gpurun_out/bench.json 2> gpurun_out/bench.err
timeout 300 compute-sanitizer --tool racecheck --racecheck-report hazard --print-limit 20 python tools/sanitize_cases.py step_c4s > gpurun_out/san/step_c4s_racecheck.txt 2>&1
timeout 300 compute-sanitizer --tool racecheck --racecheck-report hazard --print-limit 20 python tools/sanitize_cases.py lean_c4s > gpurun_out/san/lean_c4s_racecheck.txt 2>&1
timeout 300 compute-sanitizer --tool memcheck python tools/sanitize_cases.py lean_c4s lean_c1 > gpurun_out/san/lean_memcheck.txt 2>&1
cat gpurun_out/pytest_gpu.txt | cut -c1-200
grep -h "SUMMARY" gpurun_out/san/*.txt
python -c "
import json
d=json.load(open('gpurun_out/bench.json')); print('bench', d['value'], d['e2e']['value'], d['secondary']['epochs_per_image'], d['secondary']['resims_per_image'], d['secondary']['log_stops_per_image'], d['clocks'])
"; tail -3 gpurun_out/bench.err
