timeout 600 ncu --set full --clock-control none --import-source on -k regex:onesweep -s 5 -c 1 -o gpurun_out/os14 python tools/prof_radix.py 1e9 u32 2 > /dev/null 2>&1
