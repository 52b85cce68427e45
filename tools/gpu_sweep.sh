mkdir -p gpurun_out
timeout 900 python tools/sweep.py 1,2,4 8,12,16 > gpurun_out/sweep_lean.txt 2>&1
cat gpurun_out/sweep_lean.txt
