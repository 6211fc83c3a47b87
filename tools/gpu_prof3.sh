for cfg in 1 3; do
MSORT_OS_CFG=$cfg timeout 600 ncu --set full --clock-control none --import-source on -k regex:onesweep -s 5 -c 1 -o gpurun_out/os3_cfg$cfg python tools/prof_radix.py 268435456 u32 2 > /dev/null 2>&1
done
