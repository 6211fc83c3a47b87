timeout 900 python -m pytest tests/test_gpu_parity.py -q -x --timeout 600 2>&1 | tail -2
for d in uniform zipf zipf_rank normal sorted; do timeout 300 python tools/time_radix.py 2e9 u32 $d 3 | cut -c1-330; done
