#!/bin/bash
# u32 look-back window / group and keys per thread, re-checked with ld.global.cg tile loads
tools/gpu_abn.sh "base w1 w3 g16 g64 i30" "4e9 u32 uniform;2e9 f32 uniform" 3 > gpurun_out/s17_u32.txt 2>&1
