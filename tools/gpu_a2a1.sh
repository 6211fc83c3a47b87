timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_dist.py -q -x --timeout 600 2>&1 | tail -15
for g in 2 4 8; do timeout 600 python tools/time_p2p.py 1e9 $g u32 uniform 2 | cut -c1-600; done
