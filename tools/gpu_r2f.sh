#!/bin/bash
export PATH=/usr/local/cuda/bin:$PATH
timeout 1800 python -m pytest tests/test_gpu_parity.py -x -q -rs > gpurun_out/r2f_tests.txt 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"onesweep|hist_kernel|scan_kernel|fill_kernel" --csv --log-file gpurun_out/r2_launches_bench.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu --no-links > gpurun_out/r2_launches_bench.out 2>&1
timeout 600 python bench.py > gpurun_out/r2f_bench1.json 2> gpurun_out/r2f_bench1.err
