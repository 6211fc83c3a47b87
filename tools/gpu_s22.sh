#!/bin/bash
# 4-byte peer-match ranking (skewed passes): share of items ranked by the 8-ballot match vs smem atomicOr masks
tools/gpu_abn.sh "base bmall bm3of4 bm1of4 bmnone" "2e9 u32 zipf;2e9 f32 uniform;2e9 u32 normal;4e9 u32 uniform" 2 > gpurun_out/s22_bm.txt 2>&1
