timeout 240 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -p no:cacheprovider -k "test_C1_784x100_8bit_20_images or lean_kernel_selection" 2>&1 | tail -15 > gpurun_out/pytest_quick.txt
cat gpurun_out/pytest_quick.txt
