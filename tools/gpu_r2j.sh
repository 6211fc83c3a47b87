#!/bin/bash
free -g > gpurun_out/r2j_free.txt; nproc >> gpurun_out/r2j_free.txt
timeout 1200 python bench.py --steps 3 --warmup 3 --no-e2e --no-cpu --het --het-ooc-chunk 536870912 > gpurun_out/r2j_bench_ooc.json 2> gpurun_out/r2j_bench_ooc.err
