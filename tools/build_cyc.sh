# experiment build: the lean kernel's per-path cycle split in the epoch trace (tools/trace_lean.py)
mkdir -p exp_libs
cd paper_conf_date_shelm19_b200/csrc && nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 \
  -Xcompiler -fPIC,-O2,-fno-fast-math -shared --expt-relaxed-constexpr -DSNN_LEAN_TRACE_CYCLES=1 -I../../include -I. \
  -o ../../exp_libs/libsnn_cyc.so snn_kernels.cu snn_event.cu snn_lean.cu snn_infer.cu snn_sparse.cu snn_api.cu
