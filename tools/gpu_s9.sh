#!/bin/bash
# launch list of the headline bench command, this library's kernels only (torch's input generation filtered out)
export PATH=/usr/local/cuda/bin:$PATH
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k 'regex:hist_kernel|scan_kernel|onesweep_kernel|merge_pipe_kernel|partition_thread_kernel|pivot_kernel|splitter_kernel|stage_|fill_kernel|barrier_kernel|copy16_kernel|rank_probe_kernel|rank_check_keys|count_diff' -c 400 --csv --log-file gpurun_out/s9_launches_bench.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu --no-links > gpurun_out/s9_launches_bench.out 2>&1
