exec > gpurun_out/merge3.log 2>&1
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "merge or virtual or p2p" 2>&1 | tail -3
for v in 3 6 7 8 2; do
  for kt in u32 u64; do MSORT_MERGE_V=$v timeout 120 python tools/time_merge.py 2.68e8 $kt 10; done
  MSORT_MERGE_V=$v timeout 120 python tools/time_merge.py 1.07e9 u32 5
  MSORT_MERGE_V=$v timeout 120 python tools/time_merge.py 2.68e8 u32 10 0.1
done
MSORT_MERGE_V=3 timeout 600 ncu --set full --clock-control none --import-source on -k regex:merge_pipe -s 3 -c 1 -o gpurun_out/merge_v3c python tools/time_merge.py 2.68e8 u32 2 > /dev/null 2>&1
MSORT_MERGE_V=3 timeout 600 ncu --metrics gpu__time_duration.sum -k regex:partition -s 3 -c 1 python tools/time_merge.py 2.68e8 u32 2 | grep -i "duration"
timeout 300 python tools/time_p2p.py 2.68e8 2 u32
timeout 300 python tools/time_p2p.py 1e9 8 u32
timeout 300 python tools/time_p2p.py 1e9 8 u32 uniform 2
