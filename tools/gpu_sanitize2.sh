timeout 900 compute-sanitizer --tool memcheck --print-limit 6 python tools/sanitize_small.py 2>&1 | grep -vE "^(u32|f32|u64) " | head -60
