#!/bin/bash
# Timing ablations of the event engine (results of variants != 0 are WRONG by construction; per-epoch
# time is what is compared).  Build here:  tools/ablate.sh build ;  run on the GPU:  tools/ablate.sh run
set -e
cd "$(dirname "$0")/.."
CS=paper_conf_date_shelm19_b200/csrc
if [ "$1" = build ]; then
  mkdir -p exp_libs
  for v in 1 2 4; do
    nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -shared -Xcompiler -fPIC -DSNN_EXP=$v \
      -I include -I $CS -o exp_libs/libsnn_exp$v.so $CS/snn_kernels.cu $CS/snn_event.cu $CS/snn_api.cu &
  done
  wait
else
  for v in 0 1 2 4; do
    lib=paper_conf_date_shelm19_b200/libsnn_b200.so
    [ $v != 0 ] && lib=exp_libs/libsnn_exp$v.so
    [ -f $lib ] || continue
    SNN_LIB_PATH=$PWD/$lib timeout 300 python bench.py --steps 5 --warmup 3 --cpu-images 0 2>/dev/null | tail -1 | \
      python -c "import json,sys; d=json.loads(sys.stdin.read()); e=d['secondary']['epochs_per_image']; print('exp $v', round(d['value'],1), 'img/s  epochs/img', round(e,2), ' us/epoch', round(1e6/d['value']/e,2))"
  done
fi
