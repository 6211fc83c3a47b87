#!/bin/bash
tools/gpu_abn.sh "base i30 i32 i31" "4e9 u32 uniform;2e9 f32 uniform;2e9 u32 zipf" 2 > gpurun_out/r2o_ab.txt 2>&1
tools/gpu_abn.sh "base ce64" "2e9 u64 uniform" 3 >> gpurun_out/r2o_ab.txt 2>&1
