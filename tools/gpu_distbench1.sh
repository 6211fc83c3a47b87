exec > gpurun_out/distbench2.log 2>&1
for g in 2 8; do
MSORT_BENCH_SAME_GPU=1 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node $g --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus $g --steps 3 --warmup 3 --keys 1e9 > gpurun_out/db2_${g}.json 2> gpurun_out/db2_${g}.err
echo "g=$g rc=$?"; tail -c 300 gpurun_out/db2_${g}.err
python -c "import json; d=json.load(open('gpurun_out/db2_${g}.json')); print(d['value'], d['config']['exchange'], json.dumps(d['alg2']), d['e2e']['value'])"
done
