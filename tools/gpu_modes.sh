mkdir -p gpurun_out
timeout 300 python bench.py --mode ensemble --steps 5 --warmup 3 > gpurun_out/ens1.json 2> gpurun_out/modes.err
timeout 300 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29511 bench.py --gpus 2 --mode ensemble --steps 3 --warmup 3 > gpurun_out/ens2.json 2>> gpurun_out/modes.err
timeout 300 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29512 bench.py --gpus 2 --mode shard-weak --steps 2 --warmup 3 --images-per-step 4 --no-infer --cpu-images 0 > gpurun_out/sw2.json 2>> gpurun_out/modes.err
for f in ens1 ens2 sw2; do echo $f; head -c 600 gpurun_out/$f.json; echo; done; tail -5 gpurun_out/modes.err
