#!/bin/bash
# skew policy re-check with the 3-of-4 ballot peer match: MSORT_SKEW_MODE 0 (peer match), 1 (hot-4), 2 (default), 3 (plain atomics)
for r in 1 2; do
  for c in "2e9 u32 zipf" "2e9 u32 zipf_rank" "2e9 f32 uniform" "1e9 f64 uniform"; do
    for m in 0 1 2 3; do
      echo "m$m $(MSORT_SKEW_MODE=$m timeout 300 python tools/time_radix.py $c 5)"
    done
  done
done > gpurun_out/s25_skew.txt 2>&1
