timeout 900 python bench.py --steps 5 --warmup 3 --cpu-seconds 10 --het > gpurun_out/bench_r1b.json 2> gpurun_out/bench_r1b.err
tail -c 300 gpurun_out/bench_r1b.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_r1b.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:onesweep -s 6 -c 1 -o gpurun_out/bench_onesweep_r1b python tools/prof_radix.py 4e9 u32 2 > /dev/null 2>&1
timeout 900 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/bench_ref_r1b.json 2>/dev/null
