#!/bin/bash
tools/gpu_abn.sh "base i26 i30 i24 g64" "4e9 u32 uniform;2e9 f32 uniform" 2 > gpurun_out/r2n_ab.txt 2>&1
