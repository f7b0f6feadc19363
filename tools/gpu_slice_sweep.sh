#!/bin/bash
# slice-grouped insert: slices x chunk size x slices per launch (tools/rates.py, 2^28, |g| = 16)
cd $GRAFT_REPO_ROOT
O=gpurun_out/${1:-slsweep}.jsonl
: > $O
for ch in 26 28; do
  for spl in 1 0; do
    for nb in 8 16 32; do
      WD_SLICE_CHUNK_LOG2=$ch WD_SLICES_PER_LAUNCH=$spl timeout 120 python tools/rates.py 28 16 slices=$nb reps=4 | sed "s/}$/, \"chunk_log2\": $ch, \"slices_per_launch\": $spl}/" >> $O
    done
  done
done
