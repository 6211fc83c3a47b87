#!/bin/bash
# skew policy: hot-4 also when the 4 largest bins hold > 1/2 of the keys (top4) vs the default (base)
tools/gpu_abn.sh "base top4" "2e9 f32 uniform;1e9 f64 uniform;2e9 u32 zipf;2e9 u32 zipf_rank;2e9 u32 normal;4e9 u32 uniform" 2 > gpurun_out/s26_top4.txt 2>&1
