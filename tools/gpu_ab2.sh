exec > gpurun_out/ab2.log 2>&1
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x --timeout 300 -k "radix or p2p_sort_virtual or small_sort" 2>&1 | tail -1
for r in 1 2 3; do
echo "base"; MSORT_PKG_ROOT=tools/_ablate/base timeout 120 python tools/time_radix.py 4e9 u32 uniform 5 | grep -o '"pass_ms": [0-9.]*'
echo "new"; timeout 120 python tools/time_radix.py 4e9 u32 uniform 5 | grep -o '"pass_ms": [0-9.]*'
done
echo "base u64"; MSORT_PKG_ROOT=tools/_ablate/base timeout 120 python tools/time_radix.py 2e9 u64 uniform 5 | grep -o '"pass_ms": [0-9.]*'
echo "new u64"; timeout 120 python tools/time_radix.py 2e9 u64 uniform 5 | grep -o '"pass_ms": [0-9.]*'
