# hot-digit ranking for skewed passes + sanitizers on the new merge / NEXT-1 paths
exec > gpurun_out/skew1.log 2>&1
timeout 1500 python -m pytest tests -m gpu -q -x --timeout 400 2>&1 | tail -3
for d in zipf zipf_rank uniform; do echo "u32 $d"; timeout 120 python tools/time_radix.py 2e9 u32 $d 5 | grep -o '"sort_ms": [0-9.]*\|"pass_ms": [0-9.]*, "pass_gbs": [0-9.]*'; done
timeout 900 compute-sanitizer --tool memcheck --print-limit 6 python tools/sanitize_small.py 2>&1 | grep -vE "^(u32|f32|u64|merge) " | tail -8
timeout 900 compute-sanitizer --tool racecheck --print-limit 6 python tools/sanitize_small.py 2>&1 | grep -vE "^(u32|f32|u64|merge) " | tail -8
