#!/bin/bash
tools/gpu_abn.sh "base ns0 ns100 w3 u64w2" "4e9 u32 uniform;2e9 u64 uniform;2e9 u32 zipf" 2 > gpurun_out/r2l_ab.txt 2>&1
