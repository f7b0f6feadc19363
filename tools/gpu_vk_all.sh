#!/bin/bash
# (V, K) per |g| from HBM (2^28 keys, alpha 0.95): is the automatic choice still the best?
cd $GRAFT_REPO_ROOT
O=gpurun_out/vk_all.jsonl
: > $O
for cfg in "28 4" "28 4 v=4 k=2" "28 4 v=4 k=4" "28 4 v=1 k=8" "28 4 v=1 k=4" \
           "28 8" "28 8 v=8 k=2" "28 8 v=2 k=4" "28 8 v=4 k=4" \
           "28 32" "28 32 v=16 k=1" "28 32 v=16 k=2" "28 32 v=4 k=4" "28 32 v=8 k=2"; do
  timeout 120 python tools/rates.py $cfg reps=3 >> $O 2>> gpurun_out/vk_all.err
done
