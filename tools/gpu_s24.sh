#!/bin/bash
# 8-byte peer-match ranking (f64 uniform: the top passes are skewed by the exponent): share of items by ballot match
tools/gpu_abn.sh "base b5555 b36db b7777 b3def ball" "1e9 f64 uniform;2e9 u64 uniform" 2 > gpurun_out/s24_bm64.txt 2>&1
