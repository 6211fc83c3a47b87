#!/bin/bash
# look-back group size / window sweep
exec > gpurun_out/tune14.log 2>&1
for c in 4 3 5 7; do MSORT_OS_CFG=$c timeout 300 python -m pytest tests/test_gpu_parity.py -x -q -k "radix" 2>&1 | tail -1; done
for c in 4 3 5 7 2 4 3 5 7 2; do echo "u32 cfg $c"; MSORT_OS_CFG=$c timeout 120 python tools/time_radix.py 4e9 u32 uniform 5 | grep -o '"pass_ms": [0-9.]*, "pass_gbs": [0-9.]*'; done
for c in 2 3 2 3; do echo "u64 cfg $c"; MSORT_OS_CFG=$c timeout 120 python tools/time_radix.py 2e9 u64 uniform 3 | grep -o '"pass_ms": [0-9.]*, "pass_gbs": [0-9.]*'; done
for c in 2 4 3; do echo "zipf cfg $c"; MSORT_OS_CFG=$c timeout 120 python tools/time_radix.py 2e9 u32 zipf 5 | grep -o '"pass_ms": [0-9.]*, "pass_gbs": [0-9.]*'; done
for c in 2 4; do echo "1e8 cfg $c"; MSORT_OS_CFG=$c timeout 120 python tools/time_radix.py 1e8 u32 uniform 5 | grep -o '"pass_ms": [0-9.]*, "pass_gbs": [0-9.]*'; done
