timeout 900 python -m pytest tests -m gpu -q -x --timeout 300 2>&1 | tail -5
for g in 2 8; do timeout 600 python tools/time_p2p.py 1e9 $g u32 uniform 0; done
timeout 600 python tools/time_p2p.py 5e8 4 u64 uniform 0
timeout 600 ncu --set full --clock-control none --import-source on -k regex:merge_tma -s 2 -c 1 -o gpurun_out/merge_r2 python tools/time_p2p.py 268435456 2 u32 > /dev/null 2>&1
