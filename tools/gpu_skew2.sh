exec > gpurun_out/skew2.log 2>&1
for m in 0 1 2; do for d in zipf zipf_rank; do echo "mode $m $d"; MSORT_SKEW_MODE=$m timeout 120 python tools/time_radix.py 2e9 u32 $d 5 | grep -o '"sort_ms": [0-9.]*\|"pass_ms": [0-9.]*, "pass_gbs": [0-9.]*'; done; done
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "radix or distributions or virtual" 2>&1 | tail -1
timeout 1800 python -m pytest tests/test_gpu_fullsize.py -q -x --timeout 600 2>&1 | tail -3
timeout 900 python tools/run_configs.py 3 > gpurun_out/configs_r1.jsonl
cat gpurun_out/configs_r1.jsonl | cut -c1-200
