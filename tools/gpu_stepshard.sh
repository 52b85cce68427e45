# per-step engine column sharding (16/32-bit C4) + regression of the step engine and lean shards
mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_step_sharding.py tests/test_gpu_sharding.py tests/test_gpu_fp32.py tests/test_gpu_16bit.py -m gpu -q -p no:cacheprovider -x 2>&1 | tail -30 > gpurun_out/pytest_stepshard.txt
cat gpurun_out/pytest_stepshard.txt
