exec > gpurun_out/merge1.log 2>&1
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "merge or virtual or p2p" 2>&1 | tail -3
for v in 2 3 4 5; do
  for kt in u32 u64; do MSORT_MERGE_V=$v timeout 120 python tools/time_merge.py 2.68e8 $kt 10; done
  MSORT_MERGE_V=$v timeout 120 python tools/time_merge.py 1.07e9 u32 5
  MSORT_MERGE_V=$v timeout 120 python tools/time_merge.py 2.68e8 u32 10 0.1
done
MSORT_MERGE_V=4 timeout 300 python tools/time_p2p.py 2.68e8 2 u32
MSORT_MERGE_V=2 timeout 300 python tools/time_p2p.py 2.68e8 2 u32
MSORT_MERGE_V=4 timeout 300 python tools/time_p2p.py 1e9 8 u32
MSORT_MERGE_V=2 timeout 300 python tools/time_p2p.py 1e9 8 u32
