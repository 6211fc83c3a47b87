#!/bin/bash
# u64/f64 onesweep tile configurations (threads, keys per thread, blocks per SM, look-back window / group)
tools/gpu_abn.sh "base t512 t512w2 t512g8 i16 i12b5" "2e9 u64 uniform;1e9 f64 uniform" 2 > gpurun_out/s4_u64_ab.txt 2>&1
