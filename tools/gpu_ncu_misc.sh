mkdir -p gpurun_out
timeout 300 ncu --set full --clock-control none --import-source on -k infer_kernel -c 1 -o gpurun_out/infer_full -f python tools/bench_infer.py --images 1332 --steps 1 --warmup 1 > gpurun_out/ncu_infer.log 2>&1
python tools/ncu_summary.py gpurun_out/infer_full.ncu-rep gpurun_out/ncu_infer_latest.json --images 1332 --source "r01 end: ncu --set full -k infer_kernel -c 1 tools/bench_infer.py --images 1332" > /dev/null 2>&1
timeout 300 ncu --set full --clock-control none --import-source on -k sparse_kernel -c 1 -o gpurun_out/sparse_full -f python tools/bench_sparse.py --trials 592 --steps 1 > gpurun_out/ncu_sparse.log 2>&1
python tools/ncu_summary.py gpurun_out/sparse_full.ncu-rep gpurun_out/ncu_sparse_latest.json --images 592 --n-exc 1000 --source "r01 end: ncu --set full -k sparse_kernel -c 1 tools/bench_sparse.py --trials 592" > /dev/null 2>&1
timeout 120 python tools/bench_sparse.py > gpurun_out/bench_sparse.json 2>/dev/null
ls gpurun_out/*latest.json; cat gpurun_out/bench_sparse.json
