#!/bin/bash
# configs[4] key types on one GPU with traffic + smem_pipe from their own captures
exec > gpurun_out/benchc5.log 2>&1
for kt in u64 f32; do
timeout 900 python bench.py --key-type $kt --keys 2e9 --steps 5 --warmup 3 --het > gpurun_out/bench_c5_$kt.json 2> gpurun_out/bench_c5_$kt.err; echo "$kt rc $?"; tail -c 300 gpurun_out/bench_c5_$kt.err
done
