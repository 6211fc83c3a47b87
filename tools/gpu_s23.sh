#!/bin/bash
# 4-byte peer-match ranking: 2/3, 3/4, 4/5, 7/8 of the items by the ballot match
tools/gpu_abn.sh "base bm23 bm34 bm45 bm78" "2e9 u32 zipf;2e9 f32 uniform;2e9 u32 normal;2e9 u32 zipf_rank" 2 > gpurun_out/s23_bm.txt 2>&1
