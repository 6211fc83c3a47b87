./tools/cub/cub_sort_bench 1e9
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv ./tools/cub/cub_sort_bench 268435456 2>/dev/null | grep -E "Onesweep|Histogram" | head -12 > gpurun_out/cub_launches.csv
