timeout 2400 python -m pytest tests/test_gpu_fullsize.py tests/test_gpu_parity.py -q --timeout 2000 --durations=5 2>&1 | tail -12
