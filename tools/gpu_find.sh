timeout 400 python -m pytest tests/test_gpu_parity.py -m gpu -q -p no:cacheprovider -k "inh_hold_mode or undo_log or raster_input or stepwise" --timeout 60 --durations 15 2>&1 | tail -40 > gpurun_out/pytest_find.txt
cat gpurun_out/pytest_find.txt | tail -30
