#!/bin/bash
# skewed passes: hot-digit count from the histogram (hk) vs always 4 (base)
tools/gpu_abn.sh "base hk" "2e9 u32 zipf_rank;2e9 u32 zipf;2e9 u32 normal;4e9 u32 uniform" 2 > gpurun_out/s11_hotk.txt 2>&1
