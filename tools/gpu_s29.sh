#!/bin/bash
# 8-byte peer-match ranking mixes on u64 keys with a zipf high word (tools/time_radix_u64skew.py)
for r in 1 2; do for nm in base b55 b77 b77m b55m; do
  echo "$nm $(MSORT_PKG_ROOT=tools/_ablate/$nm timeout 300 python tools/time_radix_u64skew.py 1e9 5)"
done; done > gpurun_out/s29_u64skew.txt 2>&1
