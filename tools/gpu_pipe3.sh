exec > gpurun_out/pipe3.log 2>&1
timeout 600 python tools/time_e2e.py 4e9 u32 3
