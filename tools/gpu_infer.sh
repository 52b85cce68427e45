set -x
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_infer.py -m gpu -x -q -p no:cacheprovider 2>&1 | tail -25 > gpurun_out/pytest_infer.txt
timeout 300 python tools/bench_infer.py > gpurun_out/bench_infer.json 2> gpurun_out/bench_infer.err
timeout 300 python tools/bench_infer.py --membrane 1 > gpurun_out/bench_infer_fixed.json 2>> gpurun_out/bench_infer.err
timeout 300 ncu --set full --clock-control none --import-source on -k infer_kernel -c 1 -o gpurun_out/infer_full -f python tools/bench_infer.py --images 1184 --steps 1 --warmup 1 > gpurun_out/ncu_infer.log 2>&1
tail -5 gpurun_out/pytest_infer.txt; cat gpurun_out/bench_infer.json gpurun_out/bench_infer_fixed.json; tail -5 gpurun_out/bench_infer.err; tail -3 gpurun_out/ncu_infer.log
