#!/bin/bash
# insert |g| 4 (the table's) vs 8 on large A = 4 tables (where slices stop fitting the L2)
cd $GRAFT_REPO_ROOT
O=gpurun_out/r02ig
mkdir -p $O
for lg in 29 30 31; do
  for ig in 0 8; do
    timeout 300 python tools/rates.py $lg 4 0.95 ig=$ig qg=16 reps=2 >> $O/ig_large.jsonl 2>> $O/ig_large.err
  done
done
