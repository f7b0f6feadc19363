#!/bin/bash
# line-window insert: 4 (default) vs 5 blocks/SM
cd $GRAFT_REPO_ROOT
O=gpurun_out/r02t
mkdir -p $O
for rep in 1 2; do
  timeout 120 python tools/rates.py 28 16 0.95 reps=3 | sed 's|}$|, "lib": "minb4"}|' >> $O/ab.jsonl
  WD_LIBRARY=build/ab/lib_insline5.so timeout 120 python tools/rates.py 28 16 0.95 reps=3 | sed 's|}$|, "lib": "minb5"}|' >> $O/ab.jsonl
done
