#!/bin/bash
# |g| = 16, 2^28: slots per lane V x keys in flight K for the sliced insert and the retrieve
cd $GRAFT_REPO_ROOT
O=gpurun_out/${1:-vksweep}.jsonl
shift
: > $O
for vk in "${@:-8 2}"; do
  set -- $vk
  WD_SLICE_CHUNK_LOG2=28 timeout 120 python tools/rates.py 28 16 v=$1 k=$2 reps=3 >> $O
  WD_SLICE_CHUNK_LOG2=28 timeout 120 python tools/rates.py 24 16 v=$1 k=$2 reps=3 >> $O
done
