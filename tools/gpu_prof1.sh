timeout 900 python -m pytest tests -m gpu -q --timeout 300 2>&1 | tail -15 > gpurun_out/pytest_gpu.txt
tail -5 gpurun_out/pytest_gpu.txt
timeout 600 ncu --set full --clock-control none --import-source on -k regex:onesweep -s 5 -c 1 -o gpurun_out/onesweep_r1 python tools/prof_radix.py 268435456 u32 2 > gpurun_out/ncu1.log 2>&1
tail -3 gpurun_out/ncu1.log
timeout 600 ncu --set full --clock-control none --import-source on -k regex:hist -s 1 -c 1 -o gpurun_out/hist_r1 python tools/prof_radix.py 268435456 u32 2 > gpurun_out/ncu2.log 2>&1
tail -3 gpurun_out/ncu2.log
