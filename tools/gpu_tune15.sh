#!/bin/bash
# early tile claim (config 10) vs config 0, interleaved on one box; parity of config 10
exec > gpurun_out/tune15.log 2>&1
MSORT_OS_CFG=10 timeout 400 python -m pytest tests/test_gpu_parity.py -x -q -k "radix or sort" 2>&1 | tail -1
for c in 0 10 0 10 0 10; do echo "u32 cfg $c"; MSORT_OS_CFG=$c timeout 120 python tools/time_radix.py 4e9 u32 uniform 5 | grep -o '"sort_ms": [0-9.]*\|"pass_ms": [0-9.]*, "pass_gbs": [0-9.]*'; done
for c in 0 10 0 10; do echo "u64 cfg $c"; MSORT_OS_CFG=$c timeout 120 python tools/time_radix.py 2e9 u64 uniform 3 | grep -o '"sort_ms": [0-9.]*\|"pass_ms": [0-9.]*, "pass_gbs": [0-9.]*'; done
for c in 0 10; do echo "zipf cfg $c"; MSORT_OS_CFG=$c timeout 120 python tools/time_radix.py 2e9 u32 zipf 3 | grep -o '"pass_ms": [0-9.]*, "pass_gbs": [0-9.]*'; done
