exec > gpurun_out/c1b.log 2>&1
for c in 0 1 2 4 5 7 8 9; do echo "cfg $c"; MSORT_OS_CFG=$c timeout 120 python tools/time_small.py 1048576 u32 300 | head -1; done
