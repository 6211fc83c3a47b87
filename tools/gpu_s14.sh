#!/bin/bash
# on top of ld.global.cg tile loads: histogram loads .cg, u64 keys per thread / window, u32 keys per thread
tools/gpu_abn.sh "lcg lcgh lcgi16 lcgi14 lcgw1 lcgi30" "4e9 u32 uniform;2e9 u64 uniform;2e9 f32 uniform;2e9 u32 zipf" 2 > gpurun_out/s14_cg.txt 2>&1
