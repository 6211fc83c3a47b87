timeout 900 python -m pytest tests/test_gpu_dist.py -q -x --timeout 400 2>&1 | tail -15
