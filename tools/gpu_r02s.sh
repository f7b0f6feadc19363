#!/bin/bash
# slice count of the grouped insert with the session-3 grouping (2^28 pairs, |g| 16, alpha 0.95)
cd $GRAFT_REPO_ROOT
O=gpurun_out/r02s
mkdir -p $O
for rep in 1 2; do
  for sl in 0 16 32 64 128; do
    timeout 120 python tools/rates.py 28 16 0.95 slices=$sl reps=3 >> $O/slices.jsonl 2>> $O/slices.err
  done
done
