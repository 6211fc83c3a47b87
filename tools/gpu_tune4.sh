for cfg in 0 3 4; do MSORT_OS_CFG=$cfg timeout 300 python tools/time_radix.py 2e9 u32 uniform 3 | cut -c1-220; done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:onesweep -s 5 -c 1 -o gpurun_out/os13 python tools/prof_radix.py 1e9 u32 2 > /dev/null 2>&1
