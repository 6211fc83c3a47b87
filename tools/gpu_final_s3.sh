#!/bin/bash
# final check of the session-3 library on a fresh box: smoke, the GPU suite, the default bench line
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/final_smoke.txt 2>&1
python -m pytest tests -m gpu -x -q > gpurun_out/final_gpu.txt 2>&1
python bench.py > gpurun_out/final_bench.json 2> gpurun_out/final_bench.err
