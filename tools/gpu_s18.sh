#!/bin/bash
# 4-byte keys in 512-thread tiles (2 blocks/SM), re-checked with ld.global.cg tile loads
tools/gpu_abn.sh "base t512i28 t512i14 t512i20 t512i28g16" "4e9 u32 uniform;2e9 f32 uniform;2e9 u32 zipf" 2 > gpurun_out/s18_u32_512.txt 2>&1
