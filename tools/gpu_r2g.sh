#!/bin/bash
# round-2 final checks: the whole GPU suite (incl. the new full-size cases), every BASELINE config on one GPU
timeout 3000 python -m pytest tests -q -m gpu -rs > gpurun_out/r2g_tests.txt 2>&1
timeout 1500 python tools/run_configs.py 3 > gpurun_out/r2g_configs.jsonl 2> gpurun_out/r2g_configs.err
