#!/bin/bash
# experiment: persisting L2 access-policy window over the current slice (slice-grouped insert)
cd $GRAFT_REPO_ROOT
O=gpurun_out/r02l2p
mkdir -p $O
tools/l2attr > $O/l2attr.txt 2>&1
for rep in 1 2; do
  for mb in 0 40 60 80 100; do
    if [ $mb = 0 ]; then timeout 120 python tools/rates.py 28 16 0.95 reps=3 | sed "s|}$|, \"persist_mb\": 0}|" >> $O/l2p.jsonl 2>> $O/l2p.err
    else WD_L2_PERSIST=$mb timeout 120 python tools/rates.py 28 16 0.95 reps=3 | sed "s|}$|, \"persist_mb\": $mb}|" >> $O/l2p.jsonl 2>> $O/l2p.err; fi
  done
done
