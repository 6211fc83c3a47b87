#!/bin/bash
# look-back groups: u32 cfg 0 (G=8), 1 (tile walk), 2 (G=16), 4 (G=32); u64 0 (G=8), 1, 2 (G=16)
exec > gpurun_out/tune13.log 2>&1
for c in 0 1 2 4; do MSORT_OS_CFG=$c timeout 300 python -m pytest tests/test_gpu_parity.py -x -q -k "radix" 2>&1 | tail -1; done
for c in 0 1 2 4 0 1 2 4; do echo "u32 cfg $c"; MSORT_OS_CFG=$c timeout 120 python tools/time_radix.py 4e9 u32 uniform 5 | grep -o '"pass_ms": [0-9.]*, "pass_gbs": [0-9.]*'; done
for c in 0 1 2 0 1 2; do echo "u64 cfg $c"; MSORT_OS_CFG=$c timeout 120 python tools/time_radix.py 2e9 u64 uniform 3 | grep -o '"pass_ms": [0-9.]*, "pass_gbs": [0-9.]*'; done
for c in 0 1; do echo "zipf cfg $c"; MSORT_OS_CFG=$c timeout 120 python tools/time_radix.py 2e9 u32 zipf 5 | grep -o '"pass_ms": [0-9.]*, "pass_gbs": [0-9.]*'; done
for c in 0 2; do MSORT_OS_CFG=$c timeout 120 python tools/lb_stats.py 4e9 u32; done
