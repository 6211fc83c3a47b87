for tool in memcheck racecheck synccheck; do
  echo "== $tool"
  timeout 900 compute-sanitizer --tool $tool --print-limit 20 python tools/sanitize_small.py 2>&1 | grep -vE "^(u32|f32|u64) " | tail -6
done
