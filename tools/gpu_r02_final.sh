# r02 final pass: -m gpu suite, smoke, bench (all fields), reference arm, every config, C5 ensemble, NEXT-2,
# the ncu launch list of the bench command and one ncu --set full capture of the dominant kernel
mkdir -p gpurun_out/final
O=gpurun_out/final
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > $O/smi.txt
lscpu > $O/lscpu.txt 2>&1
timeout 1500 python -m pytest tests -m gpu -q -rs -p no:cacheprovider 2>&1 | tail -15 > $O/pytest_gpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.txt 2>&1
timeout 900 python bench.py > $O/bench.json 2> $O/bench.err
timeout 300 python bench.py --impl reference --steps 2 --warmup 3 > $O/bench_ref.json 2>> $O/bench.err
timeout 600 python bench.py --mode ensemble --no-infer > $O/bench_ensemble.json 2>> $O/bench.err
timeout 900 python tools/bench_configs.py > $O/configs.jsonl 2> $O/configs.err
timeout 600 python tools/bench_next2.py > $O/next2.jsonl 2> $O/next2.err
timeout 300 python tools/bench_infer.py > $O/infer.json 2> $O/infer.err
timeout 400 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches.csv python bench.py --steps 2 --warmup 3 --cpu-images 0 --no-infer --no-floor > $O/bench_ncu.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:present_lean --launch-skip 1 -c 1 -o $O/lean_full -f python tools/ncu_target.py --images 32 > $O/ncu_lean.log 2>&1
python tools/ncu_summary.py $O/lean_full.ncu-rep $O/ncu_full_latest.json --images 32 --source "r02 final: ncu --set full --clock-control none -k regex:present_lean --launch-skip 1 -c 1 tools/ncu_target.py --images 32" > $O/ncu_summary.log 2>&1
python tools/ncu_lines.py $O/lean_full.ncu-rep 40 > $O/lean_source_top.txt 2>&1
cat $O/pytest_gpu.txt | cut -c1-200; tail -2 $O/smoke.txt
python - <<'PY'
import json
O='gpurun_out/final'
d=json.load(open(f'{O}/bench.json'))
print('bench', d['value'], 'e2e', d['e2e']['value'], 'clocks', d['clocks'])
print('roofline', {k: d['roofline'][k] for k in ('achieved','peak','frac','kernel_ms_per_launch','kernel_share_of_step','alg_bytes_per_launch','traffic')})
print('floor', d['latency_roofline']['frac'], 'infer', d['inference']['value'], d['inference']['roofline']['frac'])
print('ens', open(f'{O}/bench_ensemble.json').read()[:300])
PY
tail -3 $O/bench.err; head -c 300 $O/bench_ref.json; echo; cat $O/configs.jsonl | cut -c1-220; cat $O/next2.jsonl | cut -c1-200; tail -2 $O/ncu_lean.log; cat $O/ncu_summary.log | tail -3
