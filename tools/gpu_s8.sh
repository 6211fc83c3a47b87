#!/bin/bash
# session-3 evidence: N=1 headline bench, configs[4] key types, launch list of the headline command,
# ncu --set full of one u64 pass (2e9 keys) for profiles/onesweep_traffic_u64.json
export PATH=/usr/local/cuda/bin:$PATH
python bench.py > gpurun_out/s8_bench_n1.json 2> gpurun_out/s8_bench_n1.err
python bench.py --key-type u64 --keys 2e9 --het > gpurun_out/s8_bench_u64.json 2> gpurun_out/s8_bench_u64.err
python bench.py --key-type f32 --keys 2e9 --het > gpurun_out/s8_bench_f32.json 2> gpurun_out/s8_bench_f32.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k 'regex:hist_kernel|scan_kernel|onesweep_kernel|merge_pipe_kernel|partition_thread_kernel|pivot_kernel|splitter_kernel|stage_|fill_kernel|barrier_kernel|copy16_kernel|rank_probe_kernel|rank_check_keys|count_diff' -c 400 --csv --log-file gpurun_out/s8_launches_bench.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu --no-links > gpurun_out/s8_launches_bench.out 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:onesweep -s 10 -c 1 -o gpurun_out/s8_onesweep_u64_2e9 python tools/prof_radix.py 2e9 u64 2 > gpurun_out/s8_ncu_u64.out 2>&1
