#!/bin/bash
# round-2 check: GPU suite, A/B vs round 1 (HEAD build), bench smoke at N=1 and N=2/4 sharing one GPU
timeout 2400 python -m pytest tests -x -q -m gpu > gpurun_out/r2c_tests.txt 2>&1
tools/gpu_abn.sh "base wt" "4e9 u32 uniform;2e9 u64 uniform;2e9 f32 uniform" 2 > gpurun_out/r2c_ab.txt 2>&1
timeout 600 python bench.py --keys 2.68e8 --steps 3 --warmup 3 --e2e-steps 1 --cpu-seconds 2 --het > gpurun_out/r2c_bench1.json 2> gpurun_out/r2c_bench1.err
for N in 2 4; do
MSORT_BENCH_SAME_GPU=1 timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node $N --master-addr 127.0.0.1 --master-port 2950$N bench.py --gpus $N --keys 1e9 --steps 3 --warmup 3 --e2e-steps 1 > gpurun_out/r2c_bench$N.json 2> gpurun_out/r2c_bench$N.err
done
