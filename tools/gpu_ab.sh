#!/bin/bash
# A/B timing of the working-tree library against tools/_ablate/base (tools/ab_build.py REV), same box,
# interleaved; usage: tools/gpu_ab.sh "<n kt dist>;<n kt dist>;..." ROUNDS
set -u
CASES=${1:-"4e9 u32 uniform;2e9 u64 uniform"}
ROUNDS=${2:-2}
IFS=';' read -ra CS <<< "$CASES"
for r in $(seq 1 $ROUNDS); do
  for c in "${CS[@]}"; do
    echo "B $(MSORT_PKG_ROOT=tools/_ablate/base timeout 300 python tools/time_radix.py $c 5)"
    echo "A $(timeout 300 python tools/time_radix.py $c 5)"
  done
done
