set -x
timeout 900 python bench.py --steps 5 --warmup 3 --cpu-seconds 10 > gpurun_out/bench_r1.json 2> gpurun_out/bench_r1.err
tail -2 gpurun_out/bench_r1.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_r1.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:onesweep -s 6 -c 1 -o gpurun_out/bench_onesweep_r1 python tools/prof_radix.py 4e9 u32 2 > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:hist -s 1 -c 1 -o gpurun_out/bench_hist_r1 python tools/prof_radix.py 4e9 u32 2 > /dev/null 2>&1
ls -la gpurun_out
