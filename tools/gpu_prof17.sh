exec > gpurun_out/prof17.log 2>&1
MSORT_MERGE_V=3 timeout 600 ncu --set full --clock-control none --import-source on -k regex:merge_pipe -s 3 -c 1 -o gpurun_out/merge_v3 python tools/time_merge.py 2.68e8 u32 2 > /dev/null 2>&1
MSORT_MERGE_V=3 timeout 600 ncu --set full --clock-control none --import-source on -k regex:partition -s 3 -c 1 -o gpurun_out/partition_v3 python tools/time_merge.py 2.68e8 u32 2 > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:onesweep -s 6 -c 1 -o gpurun_out/os17_u32 python tools/prof_radix.py 4e9 u32 2 > /dev/null 2>&1
ls -la gpurun_out/
