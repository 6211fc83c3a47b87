exec > gpurun_out/distbench1.log 2>&1
for g in 2 4 8; do for e in 0 2; do
MSORT_BENCH_SAME_GPU=1 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node $g --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus $g --steps 3 --warmup 3 --keys 1e9 --exchange $e > gpurun_out/db_${g}_${e}.json 2> gpurun_out/db_${g}_${e}.err
echo "g=$g e=$e rc=$?"; tail -c 200 gpurun_out/db_${g}_${e}.err
python -c "import json; d=json.load(open('gpurun_out/db_${g}_${e}.json')); print(d['value'], d['ms_per_step'], d['e2e']['value'] if d.get('e2e') else None, d['e2e'].get('phases_ms') if d.get('e2e') else None)"
done; done
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29534 bench.py --impl reference --gpus 2 --steps 2 --warmup 1 > gpurun_out/db_ref.json 2>/dev/null; echo "ref rc=$?"; head -c 300 gpurun_out/db_ref.json
