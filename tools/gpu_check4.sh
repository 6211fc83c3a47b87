# after radix epoch tags + merge defaults + fused NEXT-1
exec > gpurun_out/check4.log 2>&1
timeout 1500 python -m pytest tests -m gpu -q -x --timeout 400 2>&1 | tail -4
for c in 0 8 9 0; do echo "u32 cfg $c"; MSORT_OS_CFG=$c timeout 120 python tools/time_radix.py 4e9 u32 uniform 5 | grep -o '"sort_ms": [0-9.]*\|"pass_ms": [0-9.]*, "pass_gbs": [0-9.]*'; done
for c in 8 9; do MSORT_OS_CFG=$c timeout 300 python -m pytest tests/test_gpu_parity.py -x -q -k "radix" 2>&1 | tail -1; done
timeout 120 python tools/time_radix.py 2e9 u64 uniform 3 | grep -o '"sort_ms": [0-9.]*\|"pass_ms": [0-9.]*, "pass_gbs": [0-9.]*'
for kt in u32 u64; do timeout 120 python tools/time_merge.py 2.68e8 $kt 10; done
timeout 120 python tools/time_merge.py 1.07e9 u32 5
