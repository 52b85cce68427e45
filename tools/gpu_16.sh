mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_16bit.py -x -q -p no:cacheprovider 2>&1 | tail -30 > gpurun_out/pytest_16.txt
cat gpurun_out/pytest_16.txt
