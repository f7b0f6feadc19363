#!/bin/bash
# A/B of two library builds on the same rates configurations: tools/gpu_ab_lib.sh OUT LIB_A LIB_B [cfg ...]
cd $GRAFT_REPO_ROOT
O=gpurun_out/$1; A=$2; B=$3; shift 3
: > $O.jsonl
for rep in 1 2; do
for cfg in "$@"; do
  for lib in $A $B; do
    WD_LIBRARY=$lib timeout 120 python tools/rates.py $cfg reps=3 | sed "s|}$|, \"lib\": \"$lib\"}|" >> $O.jsonl
  done
done
done
