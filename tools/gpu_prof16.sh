#!/bin/bash
exec > gpurun_out/prof16.log 2>&1
for c in 0 0; do echo "u32 cfg $c"; MSORT_OS_CFG=$c timeout 120 python tools/time_radix.py 4e9 u32 uniform 5 | grep -o '"pass_ms": [0-9.]*, "pass_gbs": [0-9.]*'; done
for c in 0; do echo "u64 cfg $c"; MSORT_OS_CFG=$c timeout 120 python tools/time_radix.py 2e9 u64 uniform 3 | grep -o '"pass_ms": [0-9.]*, "pass_gbs": [0-9.]*'; done
timeout 120 python tools/lb_stats.py 4e9 u32
timeout 600 ncu --set full --clock-control none --import-source on -k regex:onesweep -s 6 -c 1 -o gpurun_out/os16_u32 python tools/prof_radix.py 4e9 u32 2 > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:onesweep -s 10 -c 1 -o gpurun_out/os16_u64 python tools/prof_radix.py 2e9 u64 2 > /dev/null 2>&1
