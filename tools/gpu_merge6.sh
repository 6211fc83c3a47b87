exec > gpurun_out/merge6.log 2>&1
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "merge" 2>&1 | tail -1
for v in 3 9 10 11; do
  echo "v=$v"
  for kt in u32 u64; do MSORT_MERGE_V=$v timeout 120 python tools/time_merge.py 2.68e8 $kt 10; done
  MSORT_MERGE_V=$v timeout 120 python tools/time_merge.py 1.07e9 u32 5
done
for v in 9 10 11; do MSORT_MERGE_V=$v timeout 300 python -m pytest tests/test_gpu_parity.py -q -x -k "merge" 2>&1 | tail -1; done
