#!/bin/bash
# ncu captures of the onesweep pass for u64 and f32 keys (configs[4] key types), then their bench lines
exec > gpurun_out/profkt.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:onesweep -s 6 -c 1 -o gpurun_out/os_u64 python tools/prof_radix.py 2e9 u64 2 > /dev/null 2>&1; echo "u64 rc $?"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:onesweep -s 2 -c 1 -o gpurun_out/os_f32 python tools/prof_radix.py 2e9 f32 2 > /dev/null 2>&1; echo "f32 rc $?"
ls -la gpurun_out
