#!/bin/bash
# round-2 evidence: launch list of the bench command, ncu --set full of one onesweep pass (4e9 u32) and of the
# device-resident fused stage merge (2 virtual ranks, 2^28 u32), compute-sanitizer over the new paths
export PATH=/usr/local/cuda/bin:$PATH
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/r2_launches_bench.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu --no-links > gpurun_out/r2_launches_bench.out 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:onesweep -s 6 -c 1 -o gpurun_out/r2_onesweep_4e9 python tools/prof_radix.py 4e9 u32 2 > gpurun_out/r2_ncu1.out 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:merge_pipe -s 1 -c 1 -o gpurun_out/r2_stage_merge python tools/prof_p2p.py 268435456 2 u32 0 > gpurun_out/r2_ncu2.out 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:hist_kernel -c 1 -o gpurun_out/r2_hist_4e9 python tools/prof_radix.py 4e9 u32 1 > gpurun_out/r2_ncu3.out 2>&1
bash tools/gpu_sanitize.sh
