#!/bin/bash
exec > gpurun_out/lbstats.log 2>&1
for c in 0 1 3 6 7; do MSORT_OS_CFG=$c timeout 120 python tools/lb_stats.py 4e9 u32; done
MSORT_OS_CFG=0 timeout 120 python tools/lb_stats.py 2e9 u32 zipf
