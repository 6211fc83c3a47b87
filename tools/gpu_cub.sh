#!/bin/bash
# Library context (never the product path): CUB DeviceRadixSort::SortKeys on the same B200, int and int64 offsets
nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o /tmp/cub_sort_bench tools/cub/cub_sort_bench.cu
for n in 1e9 2e9; do /tmp/cub_sort_bench $n int; /tmp/cub_sort_bench $n int64; done
