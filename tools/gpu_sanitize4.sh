# three-barrier onesweep tile (next tile counted after the scatter): memcheck / racecheck / synccheck
exec > gpurun_out/sanitize4.log 2>&1
for t in memcheck racecheck synccheck; do echo "== $t"; timeout 600 compute-sanitizer --tool $t --print-limit 6 python tools/sanitize_small.py 2>&1 | grep -vE "^(u32|f32|u64) [0-9]" | tail -15; done
