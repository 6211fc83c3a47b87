#!/bin/bash
# session-3 evidence on the final library: N>1 bench paths with ranks sharing the one GPU (correctness runs, not
# scaling numbers), the reference arm, every BASELINE config on one GPU (virtual ranks), smoke
MSORT_BENCH_SAME_GPU=1 MSORT_BENCH_FORCE_NCCL=1 timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29512 bench.py --gpus 2 --steps 3 --warmup 3 --e2e-steps 1 > gpurun_out/s16_bench2.json 2> gpurun_out/s16_bench2.err
for N in 4 8; do
MSORT_BENCH_SAME_GPU=1 timeout 1200 python -m torch.distributed.run --nnodes=1 --nproc-per-node $N --master-addr 127.0.0.1 --master-port 2952$N bench.py --gpus $N --steps 3 --warmup 3 --e2e-steps 1 > gpurun_out/s16_bench$N.json 2> gpurun_out/s16_bench$N.err
done
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/s16_bench_ref.json 2> gpurun_out/s16_bench_ref.err
timeout 1800 python tools/run_configs.py 3 > gpurun_out/s16_configs.jsonl 2> gpurun_out/s16_configs.err
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/s16_smoke.txt 2>&1
