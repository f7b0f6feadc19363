#!/bin/bash
# kF_PF A/B: hits, misses, inserts at 2^28 (HBM) and 2^20 (L2) for |g| = 1..8
cd $GRAFT_REPO_ROOT
O=gpurun_out/${1:-pf}.jsonl
: > $O
for fl in 11 27; do
  for cfg in "28 4" "28 4 q=miss" "28 8" "28 8 q=miss" "28 2" "28 1" "20 4 q=inter"; do
    timeout 120 python tools/rates.py $cfg flags=$fl reps=3 >> $O 2>> gpurun_out/${1:-pf}.err
  done
done
