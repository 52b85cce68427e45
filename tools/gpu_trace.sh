mkdir -p gpurun_out
timeout 120 python tools/trace_lean.py --images 8 > gpurun_out/trace_lean.txt 2>&1
cat gpurun_out/trace_lean.txt
