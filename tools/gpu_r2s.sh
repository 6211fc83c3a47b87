#!/bin/bash
# skewed-pass ranking modes on zipf / zipf_rank / normal (MSORT_SKEW_MODE, interleaved, same box)
for r in 1 2; do for d in zipf zipf_rank normal; do for m in 2 3 0 1; do
  echo "mode$m $(MSORT_SKEW_MODE=$m timeout 300 python tools/time_radix.py 2e9 u32 $d 5)"
done; done; done > gpurun_out/r2s_skew.txt 2>&1
