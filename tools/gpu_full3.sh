exec > gpurun_out/full3.log 2>&1
timeout 2400 python -m pytest tests/test_gpu_fullsize.py -q -x --timeout 900 -k "virtual_full_size" 2>&1 | tail -3
