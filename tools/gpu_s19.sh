#!/bin/bash
# ptxas options on the whole library: expensive optimizations, default L1 cache mode cg, -O2
tools/gpu_abn.sh "base aeo dlcm o2" "4e9 u32 uniform;2e9 u64 uniform;2e9 f32 uniform" 2 > gpurun_out/s19_ptxas.txt 2>&1
