#!/bin/bash
# register-prefetch onesweep configs vs default (u32 cfg 1,7; u64 cfg 3)
exec > gpurun_out/tune10.log 2>&1; set -x
mkdir -p gpurun_out
timeout 300 python -m pytest tests/test_gpu_parity.py -x -q -k "radix" 2>&1 | tail -3
for c in 0 1 7 0 1; do MSORT_OS_CFG=$c timeout 120 python tools/time_radix.py 4e9 u32 uniform 5; done
for c in 0 1; do MSORT_OS_CFG=$c timeout 120 python tools/time_radix.py 2e9 u32 zipf 5; done
for c in 0 3 0 3; do MSORT_OS_CFG=$c timeout 120 python tools/time_radix.py 2e9 u64 uniform 3; done
for c in 1 3; do MSORT_OS_CFG=$c MSORT_TEST_CFG=1 timeout 300 python -m pytest tests/test_gpu_parity.py -x -q -k "radix" 2>&1 | tail -2; done
