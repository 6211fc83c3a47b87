#!/bin/bash
# onesweep tile load / scatter store cache operators: ld.cs (default) / ld.cg / ld.L1::no_allocate / ld.nc; st.cs / st.cg / st.wt
tools/gpu_abn.sh "base lcg lna lg scg lcgscg swt" "4e9 u32 uniform;2e9 u64 uniform" 2 > gpurun_out/s13_cacheops.txt 2>&1
