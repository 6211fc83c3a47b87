#!/bin/bash
# skewed passes as their own kernel instantiation (HOT template flag) with the hot-digit count from the histogram
tools/gpu_abn.sh "base hot" "4e9 u32 uniform;2e9 u32 zipf_rank;2e9 u32 zipf;2e9 u32 normal;2e9 f32 uniform;2e9 u64 uniform" 2 > gpurun_out/s12_hot.txt 2>&1
