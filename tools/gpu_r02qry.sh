#!/bin/bash
# headline retrieve: 3 (default) vs 4 blocks/SM for the two-lanes-per-line query kernel
cd $GRAFT_REPO_ROOT
O=gpurun_out/r02qry
mkdir -p $O
for rep in 1 2; do
  timeout 120 python tools/rates.py 28 16 0.95 reps=3 | sed 's|}$|, "lib": "minb3"}|' >> $O/q.jsonl
  WD_LIBRARY=build/ab/lib_qry4.so timeout 120 python tools/rates.py 28 16 0.95 reps=3 | sed 's|}$|, "lib": "minb4"}|' >> $O/q.jsonl
done
