#!/bin/bash
# 4-byte peer-match ranking with a third method: __match_any_sync (ADU pipe) for some items
# mA ballot 3/4 + match 1/4; mB ballot 1/2 + match 1/2; mC ballot 1/2 + match 1/4 + atomicOr 1/4; mD ballot 1/2 + match 1/4 + atomicOr 1/4 (other order); mall match only
tools/gpu_abn.sh "base mA mB mC mD mall" "2e9 u32 zipf;2e9 u32 zipf_rank;2e9 u32 normal" 2 > gpurun_out/s27_match.txt 2>&1
