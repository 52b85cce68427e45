mkdir -p gpurun_out
timeout 200 python tools/bench_ensemble.py > gpurun_out/bench_ensemble.json 2> gpurun_out/bench_ensemble.err
timeout 200 python tools/bench_ensemble.py --nets 24 > gpurun_out/bench_ensemble24.json 2>> gpurun_out/bench_ensemble.err
cat gpurun_out/bench_ensemble.json gpurun_out/bench_ensemble24.json; tail -3 gpurun_out/bench_ensemble.err
