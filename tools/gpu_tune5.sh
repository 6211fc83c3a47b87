for cfg in 0 1 2 3; do MSORT_OS_CFG=$cfg timeout 300 python tools/time_radix.py 1e9 u64 uniform 3 | cut -c1-230; done
MSORT_OS_CFG=0 timeout 300 python tools/time_radix.py 2e9 f32 uniform 3 | cut -c1-230
