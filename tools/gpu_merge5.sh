exec > gpurun_out/merge5.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_dist.py -q -x 2>&1 | tail -3
for kt in u32 u64; do timeout 120 python tools/time_merge.py 2.68e8 $kt 10; done
timeout 120 python tools/time_merge.py 1.07e9 u32 5
timeout 120 python tools/time_merge.py 2.68e8 u32 10 0.1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:merge_pipe -s 3 -c 1 -o gpurun_out/merge_v3e python tools/time_merge.py 2.68e8 u32 2 > /dev/null 2>&1
