mkdir -p gpurun_out
SNN_LIB_PATH=exp_libs/libsnn_trace.so timeout 60 python tools/trace_lean.py --images 8 > gpurun_out/trace_lean.txt 2>&1
timeout 60 python tools/trace_lean.py --images 8 > gpurun_out/trace_lean_notcycles.txt 2>&1
cat gpurun_out/trace_lean.txt; echo ---; cat gpurun_out/trace_lean_notcycles.txt
