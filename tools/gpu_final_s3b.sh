#!/bin/bash
# final check after the skew-path changes: smoke, GPU suite, default bench, configs[4] key types, every config on one GPU
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/fb_smoke.txt 2>&1
python -m pytest tests -m gpu -x -q > gpurun_out/fb_gpu.txt 2>&1
python bench.py > gpurun_out/fb_bench.json 2> gpurun_out/fb_bench.err
python bench.py --key-type f32 --keys 2e9 --het > gpurun_out/fb_bench_f32.json 2> gpurun_out/fb_bench_f32.err
python bench.py --key-type u64 --keys 2e9 --het > gpurun_out/fb_bench_u64.json 2> gpurun_out/fb_bench_u64.err
timeout 1800 python tools/run_configs.py 3 2> gpurun_out/fb_configs.err | grep -v "^NCCL version" > gpurun_out/fb_configs.jsonl
