# ncu --set full of one 32-image C4 present_batch launch (lean kernel) -> profiles/ncu_full_latest.json (bench traffic)
mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k regex:present_lean --launch-skip 1 -c 1 -o gpurun_out/full -f python tools/ncu_target.py --images 32 > gpurun_out/ncu_full.log 2>&1
python tools/ncu_summary.py gpurun_out/full.ncu-rep gpurun_out/ncu_full_latest.json --images 32 --source "r02: ncu --set full --clock-control none -k regex:present_lean --launch-skip 1 -c 1 tools/ncu_target.py --images 32" > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:infer_kernel -c 1 -o gpurun_out/infer_full -f python tools/bench_infer.py --images 1332 > gpurun_out/ncu_infer.log 2>&1
python tools/ncu_summary.py gpurun_out/infer_full.ncu-rep gpurun_out/r02_infer_ncu_full.json --images 1332 --source "r02: ncu --set full -k regex:infer_kernel -c 1 tools/bench_infer.py --images 1332" > /dev/null 2>&1
python -c "
import json
d=json.load(open('gpurun_out/ncu_full_latest.json')); print('lean', d['dram_bytes_per_launch'], d['metrics'].get('gpu__time_duration.sum'), d['metrics'].get('launch__registers_per_thread'), d['metrics'].get('smsp__issue_active.avg.pct_of_peak_sustained_active'))
d=json.load(open('gpurun_out/r02_infer_ncu_full.json')); print('infer', d['dram_bytes_per_launch'], d['metrics'].get('gpu__time_duration.sum'))
"; tail -2 gpurun_out/ncu_full.log gpurun_out/ncu_infer.log
