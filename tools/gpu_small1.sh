exec > gpurun_out/small1.log 2>&1
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x --timeout 300 2>&1 | tail -2
timeout 300 python tools/time_small.py 1048576 u32 300
timeout 300 python tools/time_small.py 4194304 u32 200
timeout 300 python tools/time_small.py 1048576 u64 200
