#!/bin/bash
# queries with a wider (or narrower) |g| than the table's: hits, misses, config 1
cd $GRAFT_REPO_ROOT
O=gpurun_out/r02n
mkdir -p $O
for G in 1 2 32; do
  for q in x miss; do
    for qg in $G 8 16; do
      timeout 300 python tools/rates.py 28 $G 0.95 q=$q qg=$qg reps=3 >> $O/qg2.jsonl 2>> $O/qg2.err
    done
  done
done
for qg in 4 8 16 32; do
  timeout 300 python tools/rates.py 20 4 0.95 q=inter qg=$qg reps=5 >> $O/qg2.jsonl 2>> $O/qg2.err
  timeout 300 python tools/rates.py 22 8 0.95 q=inter qg=$qg reps=5 >> $O/qg2.jsonl 2>> $O/qg2.err
done
