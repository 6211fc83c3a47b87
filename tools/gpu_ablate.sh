#!/bin/bash
# onesweep timing ablations (tools/ablate_build.py): 0 = real, 1 = no look-back, 2 = no early counts, 3 = both
exec > gpurun_out/ablate.log 2>&1
for k in ${ABL:-0 1 2 3}; do
  for c in 0 1; do
    if [ $k = 0 ]; then R=""; else R=$PWD/tools/_ablate/$k; fi
    echo "ablate=$k cfg=$c"; MSORT_PKG_ROOT=$R MSORT_OS_CFG=$c timeout 120 python tools/time_radix.py 4e9 u32 uniform 5 | cut -c1-300
  done
done
