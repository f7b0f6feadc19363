#!/bin/bash
# sliced insert probe: 3 vs 4 blocks/SM (V = 16, K = 1), and K = 2 keys per lane
cd $GRAFT_REPO_ROOT
O=gpurun_out/r02q
mkdir -p $O
for rep in 1 2; do
  timeout 120 python tools/rates.py 28 16 0.95 reps=3 | sed 's|}$|, "lib": "default"}|' >> $O/ab.jsonl
  WD_LIBRARY=build/ab/lib_ins16_4.so timeout 120 python tools/rates.py 28 16 0.95 reps=3 | sed 's|}$|, "lib": "ins16_minb4"}|' >> $O/ab.jsonl
  timeout 120 python tools/rates.py 28 16 0.95 k=2 reps=3 | sed 's|}$|, "lib": "default"}|' >> $O/ab.jsonl
done
