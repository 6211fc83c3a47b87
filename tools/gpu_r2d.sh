#!/bin/bash
# round-2: new GPU tests (NCCL swap, per-stage parity, ragged chunks, out-of-core HET, dist NCCL), then the
# default bench at N=1 (full 4e9) with the HET leg, and N=2 sharing one GPU
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_het.py tests/test_gpu_dist.py -x -q > gpurun_out/r2d_tests.txt 2>&1
timeout 900 python bench.py --het > gpurun_out/r2d_bench1.json 2> gpurun_out/r2d_bench1.err
MSORT_BENCH_SAME_GPU=1 timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29502 bench.py --gpus 2 --steps 5 --warmup 3 --e2e-steps 1 > gpurun_out/r2d_bench2.json 2> gpurun_out/r2d_bench2.err
bash tools/gpu_cub.sh > gpurun_out/r2d_cub.txt 2>&1
