#!/bin/bash
tools/gpu_abn.sh "base v1 v1w4 v1w1" "4e9 u32 uniform;2e9 u64 uniform" 2 > gpurun_out/r2b_ab.txt 2>&1
