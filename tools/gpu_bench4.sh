# round-1 evidence refresh: bench line, reference arm, launch list, ncu captures of onesweep / merge / hist
timeout 900 python bench.py --steps 10 --warmup 3 --cpu-seconds 10 --het > gpurun_out/bench_r1c.json 2> gpurun_out/bench_r1c.err
tail -c 400 gpurun_out/bench_r1c.err
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/bench_ref_r1c.json 2>/dev/null
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_r1c.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:onesweep -s 6 -c 1 -o gpurun_out/os_r1c python tools/prof_radix.py 4e9 u32 2 > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:hist_kernel -s 1 -c 1 -o gpurun_out/hist_r1c python tools/prof_radix.py 4e9 u32 2 > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:merge_pipe -s 3 -c 1 -o gpurun_out/merge_r1c python tools/time_merge.py 2.68e8 u32 2 > /dev/null 2>&1
timeout 300 python tools/time_p2p.py 2.68e8 2 u32 > gpurun_out/p2p_r1c.jsonl
for g in 4 8; do for e in 0 2; do timeout 300 python tools/time_p2p.py 1e9 $g u32 uniform $e >> gpurun_out/p2p_r1c.jsonl; done; done
timeout 300 python tools/time_p2p.py 2e9 8 u32 reverse 0 >> gpurun_out/p2p_r1c.jsonl
timeout 300 python tools/time_p2p.py 2e9 8 u32 sorted 0 >> gpurun_out/p2p_r1c.jsonl
timeout 300 python tools/time_p2p.py 2e9 8 u32 zipf 0 >> gpurun_out/p2p_r1c.jsonl
head -c 300 gpurun_out/bench_r1c.json
