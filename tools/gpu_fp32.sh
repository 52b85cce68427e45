# NEXT-2 fp32 conductance: GPU parity + the 16-bit/step-engine regression subset
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_fp32.py tests/test_gpu_16bit.py -m gpu -q -p no:cacheprovider -x 2>&1 | tail -30 > gpurun_out/pytest_fp32.txt
cat gpurun_out/pytest_fp32.txt
