#!/bin/bash
# onesweep tile-shape A/B: 512-thread blocks (2 per SM) vs the 256-thread default (4 per SM)
tools/gpu_abn.sh "base t512 t512i24 t512g16" "4e9 u32 uniform;2e9 f32 uniform;2e9 u32 zipf" 2 > gpurun_out/r2h_ab.txt 2>&1
