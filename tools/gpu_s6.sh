#!/bin/bash
# u64/f64: 512-thread tiles, window 2, next tile counted after the scatter, keys per thread
tools/gpu_abn.sh "base ce cei16 cei15 cew1" "2e9 u64 uniform;1e9 f64 uniform" 3 > gpurun_out/s6_u64_ab.txt 2>&1
