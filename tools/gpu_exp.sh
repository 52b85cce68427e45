mkdir -p gpurun_out
for v in base NOATOM NOLOG BOTH; do
  if [ $v = base ]; then L=""; else L="SNN_LIB_PATH=exp_libs/lib_$v.so"; fi
  env $L timeout 120 python bench.py --steps 10 --cpu-images 0 --no-infer > gpurun_out/exp_$v.json 2>/dev/null
  python -c "import json; d=json.load(open('gpurun_out/exp_$v.json')); print('$v', d['value'])"
done
