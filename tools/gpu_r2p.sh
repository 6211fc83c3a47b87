#!/bin/bash
# round-2 final evidence on the final library: the full GPU suite, smoke, bench N=1 (defaults + HET), configs[4] u64
timeout 3000 python -m pytest tests -q -m gpu -rs > gpurun_out/r2p_tests.txt 2>&1
python __graft_entry__.py smoke >> gpurun_out/r2p_tests.txt 2>&1
timeout 900 python bench.py --het > gpurun_out/r2p_bench1.json 2> gpurun_out/r2p_bench1.err
timeout 900 python bench.py --key-type u64 --keys 2e9 --steps 5 --warmup 3 --het > gpurun_out/r2p_bench_u64.json 2> gpurun_out/r2p_bench_u64.err
