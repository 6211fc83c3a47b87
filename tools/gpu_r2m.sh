#!/bin/bash
tools/gpu_abn.sh "base u64w2 u64w1 u64w2g32 u64w2g8" "2e9 u64 uniform;1e9 f64 uniform" 3 > gpurun_out/r2m_ab.txt 2>&1
