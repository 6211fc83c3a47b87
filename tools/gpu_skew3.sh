exec > gpurun_out/skew3.log 2>&1
for m in 1 0; do for d in zipf zipf_rank; do echo "mode $m $d"; MSORT_SKEW_MODE=$m timeout 120 python tools/time_radix.py 2e9 u32 $d 5 | grep -o '"sort_ms": [0-9.]*\|"pass_ms": [0-9.]*, "pass_gbs": [0-9.]*'; done; done
echo "f32 uniform"; timeout 120 python tools/time_radix.py 2e9 f32 uniform 5 | grep -o '"sort_ms": [0-9.]*\|"pass_ms": [0-9.]*, "pass_gbs": [0-9.]*'
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x 2>&1 | tail -1
timeout 1800 python -m pytest tests/test_gpu_fullsize.py -q -x --timeout 600 -k "zipf" 2>&1 | tail -1
