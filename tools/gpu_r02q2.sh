#!/bin/bash
# headline queries (2^28, |g| 16, alpha 0.95): lanes per window (V) x keys in flight (K)
cd $GRAFT_REPO_ROOT
O=gpurun_out/r02q2
mkdir -p $O
for vk in "8 2" "16 1" "16 2" "8 4" "4 4" "4 2"; do
  set -- $vk
  timeout 120 python tools/rates.py 28 16 0.95 v=$1 k=$2 qg=16 reps=3 >> $O/vk.jsonl 2>> $O/vk.err
done
