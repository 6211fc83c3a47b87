exec > gpurun_out/numa.log 2>&1
nvidia-smi topo -m 2>&1 | head -5; lscpu | grep -E "NUMA|Socket|Model name" 
for r in 1 2; do
timeout 600 python tools/time_e2e.py 4e9 u32 2 numa
timeout 600 python tools/time_e2e.py 4e9 u32 2
done
