#!/bin/bash
# final check of the final library: full GPU suite, smoke, default bench
timeout 3000 python -m pytest tests -q -m gpu -rs > gpurun_out/r2u_tests.txt 2>&1
python __graft_entry__.py smoke >> gpurun_out/r2u_tests.txt 2>&1
timeout 900 python bench.py > gpurun_out/r2u_bench1.json 2> gpurun_out/r2u_bench1.err
