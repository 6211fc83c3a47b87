for g in 2 4 8; do timeout 600 python tools/time_p2p.py 1e9 $g u32 uniform 0; done
timeout 600 python tools/time_p2p.py 1e9 8 u32 reverse 0
timeout 600 python tools/time_p2p.py 1e9 2 u32 uniform 1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:merge_kernel -s 2 -c 1 -o gpurun_out/merge_r1 python tools/time_p2p.py 268435456 2 u32 > /dev/null 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv python tools/time_p2p.py 268435456 4 u32 2>/dev/null | grep -v "^==" > gpurun_out/p2p4_launches.csv
