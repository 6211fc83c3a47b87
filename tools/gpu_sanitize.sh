#!/bin/bash
# compute-sanitizer memcheck / racecheck / synccheck over tools/sanitize_small.py (small sorts of every path)
exec > gpurun_out/sanitize.log 2>&1
for t in memcheck racecheck synccheck; do echo "== $t"; timeout 900 compute-sanitizer --tool $t --print-limit 6 python tools/sanitize_small.py 2>&1 | grep -vE "^(u32|f32|u64) [0-9]" | tail -15; done
