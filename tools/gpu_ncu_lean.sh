mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k regex:present_lean --launch-skip 1 -c 1 -o gpurun_out/lean_full -f python tools/ncu_target.py --images 8 > gpurun_out/ncu_lean.log 2>&1
ncu -i gpurun_out/lean_full.ncu-rep --page source --csv --print-source sass > gpurun_out/lean_source_sass.csv 2>/dev/null
ncu -i gpurun_out/lean_full.ncu-rep --page source --csv > gpurun_out/lean_source_cuda.csv 2>/dev/null
ncu -i gpurun_out/lean_full.ncu-rep --page raw --csv > gpurun_out/lean_raw.csv 2>/dev/null
ls -la gpurun_out; tail -3 gpurun_out/ncu_lean.log
