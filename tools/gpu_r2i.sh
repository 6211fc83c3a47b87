#!/bin/bash
# N>1 bench on one GPU: N=2 with the NCCL leg forced (NCCL refuses two ranks on one GPU: the leg must report
# "unavailable" and the run must finish), N=4 and N=8; configs[4] key types at N=1
MSORT_BENCH_SAME_GPU=1 MSORT_BENCH_FORCE_NCCL=1 timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29512 bench.py --gpus 2 --steps 3 --warmup 3 --e2e-steps 1 > gpurun_out/r2i_bench2.json 2> gpurun_out/r2i_bench2.err
for N in 4 8; do
MSORT_BENCH_SAME_GPU=1 timeout 1200 python -m torch.distributed.run --nnodes=1 --nproc-per-node $N --master-addr 127.0.0.1 --master-port 2952$N bench.py --gpus $N --steps 3 --warmup 3 --e2e-steps 1 > gpurun_out/r2i_bench$N.json 2> gpurun_out/r2i_bench$N.err
done
timeout 900 python bench.py --key-type u64 --keys 2e9 --steps 5 --warmup 3 --het > gpurun_out/r2i_bench_u64.json 2> gpurun_out/r2i_bench_u64.err
timeout 900 python bench.py --key-type f32 --keys 2e9 --steps 5 --warmup 3 --het > gpurun_out/r2i_bench_f32.json 2> gpurun_out/r2i_bench_f32.err
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/r2i_bench_ref.json 2> gpurun_out/r2i_bench_ref.err
