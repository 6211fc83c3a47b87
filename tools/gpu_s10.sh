#!/bin/bash
# skewed passes: hot-k ranking (k = 1, 2, 4 most frequent digit values with one atomic per row) forced on every
# skewed pass (MSORT_SKEW_MODE=1) vs the default policy (mode 2) and peer match (mode 0)
for r in 1 2; do
  for c in "2e9 u32 zipf" "2e9 u32 zipf_rank" "2e9 u32 normal"; do
    echo "h4.m2 $(MSORT_PKG_ROOT=tools/_ablate/h4 MSORT_SKEW_MODE=2 timeout 300 python tools/time_radix.py $c 5)"
    echo "h4.m0 $(MSORT_PKG_ROOT=tools/_ablate/h4 MSORT_SKEW_MODE=0 timeout 300 python tools/time_radix.py $c 5)"
    for nm in h1 h2 h4; do
      echo "$nm.m1 $(MSORT_PKG_ROOT=tools/_ablate/$nm MSORT_SKEW_MODE=1 timeout 300 python tools/time_radix.py $c 5)"
    done
  done
done > gpurun_out/s10_skew.txt 2>&1
