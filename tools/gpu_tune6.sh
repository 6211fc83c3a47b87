timeout 900 python -m pytest tests -m gpu -q -x --timeout 600 2>&1 | tail -3
for cfg in 0; do MSORT_OS_CFG=$cfg timeout 300 python tools/time_radix.py 2e9 u32 uniform 3 | cut -c1-330; done
timeout 300 python tools/time_radix.py 1e9 u64 uniform 3 | cut -c1-330
