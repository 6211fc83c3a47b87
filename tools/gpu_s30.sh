#!/bin/bash
# hot-path ranking (dominant digits): share of items whose peers come from match.any (1/4, 1/3, 1/2, all) vs 4 ballots
tools/gpu_abn.sh "base h4 h3 h2 hall" "2e9 f32 uniform;2e9 u32 zipf_rank;4e9 u32 uniform;1e9 f64 uniform" 2 > gpurun_out/s30_hot.txt 2>&1
