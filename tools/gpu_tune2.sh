timeout 900 python -m pytest tests -m gpu -q -x --timeout 300 2>&1 | tail -5
for cfg in 0 1 2 3; do
  MSORT_OS_CFG=$cfg timeout 300 python tools/time_radix.py 1e9 u32 uniform
  MSORT_OS_CFG=$cfg timeout 300 python tools/time_radix.py 5e8 u64 uniform
done
MSORT_OS_CFG=1 timeout 300 python tools/time_radix.py 1e9 u32 zipf
MSORT_OS_CFG=1 timeout 600 ncu --set full --clock-control none --import-source on -k regex:onesweep -s 5 -c 1 -o gpurun_out/os12_cfg1 python tools/prof_radix.py 268435456 u32 2 > /dev/null 2>&1
