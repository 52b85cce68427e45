timeout 900 python -m pytest tests -m gpu -x -q -p no:cacheprovider 2>&1 | tail -25 > gpurun_out/pytest_lean.txt
timeout 300 python bench.py --steps 10 --cpu-images 0 > gpurun_out/bench_lean.json 2> gpurun_out/bench_lean.err
timeout 300 ncu --set full --clock-control none --import-source on -k regex:present_lean -c 1 -o gpurun_out/lean_full -f python tools/ncu_target.py --images 4 > gpurun_out/ncu_lean.log 2>&1
tail -5 gpurun_out/pytest_lean.txt; cat gpurun_out/bench_lean.json; tail -3 gpurun_out/bench_lean.err; tail -3 gpurun_out/ncu_lean.log
