#!/bin/bash
# u64/f64 onesweep tile configurations (threads, keys per thread, blocks per SM, look-back window / group)
tools/gpu_abn.sh "t512w2 t512w3 t512w4 t512w2g32 t512w2i16 t512w2ce i16w2" "2e9 u64 uniform;1e9 f64 uniform" 2 > gpurun_out/s5_u64_ab.txt 2>&1
