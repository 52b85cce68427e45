# r02 first GPU pass: full -m gpu suite (incl. the new batch-vs-oracle tests), bench, sanitizers
mkdir -p gpurun_out/san
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi.txt
timeout 1200 python -m pytest tests -m gpu -q -p no:cacheprovider -x 2>&1 | tail -15 > gpurun_out/pytest_gpu.txt
timeout 600 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err
for c in $(python tools/sanitize_cases.py --list); do
  for tool in memcheck racecheck synccheck; do
    extra=""; [ $tool = racecheck ] && extra="--racecheck-report hazard"
    timeout 600 compute-sanitizer --tool $tool $extra --print-limit 20 python tools/sanitize_cases.py $c > gpurun_out/san/${c}_${tool}.txt 2>&1
    echo "$c $tool rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY' gpurun_out/san/${c}_${tool}.txt | tail -1)" >> gpurun_out/san/summary.txt
  done
done
cat gpurun_out/pytest_gpu.txt | cut -c1-200
cat gpurun_out/san/summary.txt
python -c "
import json
d=json.load(open('gpurun_out/bench.json')); print('bench', d['value'], d['e2e']['value'], d['roofline']['frac'], d['inference']['value'], d['clocks'])
"; tail -3 gpurun_out/bench.err
