exec > gpurun_out/a2a2.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_dist.py -q -x 2>&1 | tail -3
for e in 0 2 3; do timeout 300 python tools/time_p2p.py 1e9 8 u32 uniform $e; done
for e in 0 2 3; do timeout 300 python tools/time_p2p.py 1e9 4 u32 uniform $e; done
for e in 0 2; do timeout 300 python tools/time_p2p.py 2.68e8 2 u32 uniform $e; done
