#!/bin/bash
# experiment: evict-first L2 policy on the sliced insert's streamed input (-DWD_INPUT_EVICT_FIRST)
cd $GRAFT_REPO_ROOT
O=gpurun_out/r02ef
mkdir -p $O
for rep in 1 2; do
  timeout 120 python tools/rates.py 28 16 0.95 reps=3 | sed 's|}$|, "lib": "default"}|' >> $O/ef.jsonl
  WD_LIBRARY=build/ab/lib_evict.so timeout 120 python tools/rates.py 28 16 0.95 reps=3 | sed 's|}$|, "lib": "evict_first"}|' >> $O/ef.jsonl
done
