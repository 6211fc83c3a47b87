#!/bin/bash
# 4-byte peer-match ranking, ballot match + match.any only: share of match.any items 1/3, 1/4, 1/5, 1/8
tools/gpu_abn.sh "mA m3 m5 m8" "2e9 u32 zipf;2e9 u32 zipf_rank;2e9 f32 uniform;2e9 u32 normal" 2 > gpurun_out/s28_match.txt 2>&1
