#!/bin/bash
# after ld.global.cg tile loads: GPU suite, ncu --set full of one u32 pass (4e9) and one u64 pass (2e9), headline bench
export PATH=/usr/local/cuda/bin:$PATH
python -m pytest tests -m gpu -x -q > gpurun_out/s15_gpu.txt 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:onesweep -s 6 -c 1 -o gpurun_out/s15_onesweep_4e9 python tools/prof_radix.py 4e9 u32 2 > gpurun_out/s15_ncu1.out 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:onesweep -s 10 -c 1 -o gpurun_out/s15_onesweep_u64_2e9 python tools/prof_radix.py 2e9 u64 2 > gpurun_out/s15_ncu2.out 2>&1
python bench.py > gpurun_out/s15_bench_n1.json 2> gpurun_out/s15_bench_n1.err
python bench.py --key-type u64 --keys 2e9 --het > gpurun_out/s15_bench_u64.json 2> gpurun_out/s15_bench_u64.err
python bench.py --key-type f32 --keys 2e9 --het > gpurun_out/s15_bench_f32.json 2> gpurun_out/s15_bench_f32.err
