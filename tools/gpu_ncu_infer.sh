mkdir -p gpurun_out
timeout 300 ncu --set full --clock-control none --import-source on -k infer_kernel -c 1 -o gpurun_out/infer_full -f python tools/bench_infer.py --images 1184 --steps 1 --warmup 1 > gpurun_out/ncu_infer.log 2>&1
tail -3 gpurun_out/ncu_infer.log
