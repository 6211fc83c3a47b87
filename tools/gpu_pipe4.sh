exec > gpurun_out/pipe4.log 2>&1
timeout 600 python bench.py --steps 3 --warmup 3 --no-cpu --e2e-steps 3 > gpurun_out/bench_pipe4.json 2> gpurun_out/bench_pipe4.err
tail -c 300 gpurun_out/bench_pipe4.err
python -c "import json; d=json.load(open('gpurun_out/bench_pipe4.json')); print(d['value'], json.dumps(d['e2e']))"
timeout 600 python tools/time_e2e.py 4e9 u32 2
