mkdir -p gpurun_out
SNN_LIB_PATH=exp_libs/libsnn_cyc.so timeout 120 python tools/trace_lean.py --images 8 > gpurun_out/trace_lean.txt 2>&1
timeout 120 python tools/trace_lean.py --images 8 > gpurun_out/trace_lean_nocycles.txt 2>&1
cat gpurun_out/trace_lean.txt; echo ---; cat gpurun_out/trace_lean_nocycles.txt
