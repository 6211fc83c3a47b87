#!/bin/bash
# three-barrier tile: look-back window 4 (cfg 11) and groups of 16 (cfg 12) vs config 0, interleaved
exec > gpurun_out/tune17.log 2>&1
for c in 11 12; do MSORT_OS_CFG=$c timeout 300 python -m pytest tests/test_gpu_parity.py -x -q -k "radix" 2>&1 | tail -1; done
for c in 0 11 12 0 11 12 0 11 12; do echo "u32 cfg $c"; MSORT_OS_CFG=$c timeout 120 python tools/time_radix.py 4e9 u32 uniform 5 | grep -o '"pass_ms": [0-9.]*, "pass_gbs": [0-9.]*'; done
