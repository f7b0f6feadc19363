#!/bin/bash
# insert |g| 8 vs 16 on A = 4 tables (2^28 HBM, 2^22 and 2^20 L2-resident)
cd $GRAFT_REPO_ROOT
O=gpurun_out/r02y
mkdir -p $O
for a in 0.8 0.95 0.99; do
  for ig in 8 16; do
    timeout 120 python tools/rates.py 28 4 $a ig=$ig qg=16 reps=3 >> $O/ig.jsonl 2>> $O/ig.err
  done
done
for lg in 20 22 24; do
  for ig in 8 16; do
    timeout 120 python tools/rates.py $lg 4 0.95 ig=$ig qg=16 reps=10 >> $O/ig.jsonl 2>> $O/ig.err
  done
done
