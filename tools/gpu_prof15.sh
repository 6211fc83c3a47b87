#!/bin/bash
# ncu full capture: u64 onesweep (stable atomic-ranked pass) and the new u32 default (prefetch)
timeout 600 ncu --set full --clock-control none --import-source on -k regex:onesweep -s 10 -c 1 -o gpurun_out/os15_u64 python tools/prof_radix.py 5e8 u64 2 > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:onesweep -s 5 -c 1 -o gpurun_out/os15_u32 python tools/prof_radix.py 1e9 u32 2 > /dev/null 2>&1
ls -la gpurun_out/
