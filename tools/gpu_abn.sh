#!/bin/bash
# interleaved timing of several builds under tools/_ablate/<name>: tools/gpu_abn.sh "names" "cases" ROUNDS
set -u
NAMES=$1; CASES=$2; ROUNDS=${3:-2}
IFS=';' read -ra CS <<< "$CASES"
for r in $(seq 1 $ROUNDS); do
  for c in "${CS[@]}"; do
    for nm in $NAMES; do
      echo "$nm $(MSORT_PKG_ROOT=tools/_ablate/$nm timeout 300 python tools/time_radix.py $c 5)"
    done
  done
done
