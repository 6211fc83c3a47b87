#!/bin/bash
# ceilings of the u32 onesweep pass: no global key loads / no look-back / neither
tools/gpu_abn.sh "base fl nolb both" "4e9 u32 uniform" 2 > gpurun_out/s1_ceiling.txt 2>&1
