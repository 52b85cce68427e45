# One GPU round: parity tests, smoke, bench (no profiler), launch list, one ncu --set full capture.
set -x
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 900 python -m pytest tests -m gpu -x -q -p no:cacheprovider 2>&1 | tail -25 > gpurun_out/pytest_gpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.txt 2>&1
timeout 600 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 3 --images-per-step 8 --cpu-images 0 > gpurun_out/bench_ncu.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:present_ --launch-skip 1 -c 1 -o gpurun_out/full -f python tools/ncu_target.py --images 32 > gpurun_out/ncu_full.log 2>&1
tail -3 gpurun_out/pytest_gpu.txt; cat gpurun_out/smoke.txt; cat gpurun_out/bench.json; tail -3 gpurun_out/bench.err
python tools/ncu_summary.py gpurun_out/full.ncu-rep gpurun_out/ncu_full_latest.json --images 32 --source "tools/gpu_full.sh" > /dev/null 2>&1
