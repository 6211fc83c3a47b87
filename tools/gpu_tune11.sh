#!/bin/bash
# early look-back window configs (3, 6, 7) vs 0/1
exec > gpurun_out/tune11.log 2>&1
for c in 0 1 3 6 7 0 1 3 6 7; do echo "cfg $c"; MSORT_OS_CFG=$c timeout 120 python tools/time_radix.py 4e9 u32 uniform 5 | grep -o '"pass_ms": [0-9.]*, "pass_gbs": [0-9.]*'; done
for c in 0 3 6; do echo "zipf cfg $c"; MSORT_OS_CFG=$c timeout 120 python tools/time_radix.py 2e9 u32 zipf 5 | grep -o '"pass_ms": [0-9.]*, "pass_gbs": [0-9.]*'; done
for c in 3 6 7; do MSORT_OS_CFG=$c timeout 300 python -m pytest tests/test_gpu_parity.py -x -q -k "radix" 2>&1 | tail -1; done
