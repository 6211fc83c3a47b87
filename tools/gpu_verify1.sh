exec > gpurun_out/verify1.log 2>&1
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 1500 python -m pytest tests -m gpu -q -x --timeout 900 2>&1 | tail -5
timeout 600 python bench.py --steps 10 --warmup 3 --cpu-seconds 10 > gpurun_out/bench_v1.json 2> gpurun_out/bench_v1.err
tail -c 300 gpurun_out/bench_v1.err
cat gpurun_out/bench_v1.json
