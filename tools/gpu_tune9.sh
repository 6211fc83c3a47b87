for cfg in 0 1 2 3 4 5 6 7; do MSORT_OS_CFG=$cfg timeout 300 python tools/time_radix.py 2e9 u32 uniform 3 | cut -c1-330; done
