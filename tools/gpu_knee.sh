#!/bin/bash
cd $GRAFT_REPO_ROOT
O=gpurun_out/knee.jsonl
: > $O
for cfg in "29 16 0.5 slices=1" "29 16 0.5 slices=16" "29 16 0.5 slices=32" "28 16 0.5 slices=1" "28 16 0.5 slices=16" "30 16 0.5 slices=1" "30 16 0.5 slices=32" "29 16 0.95 slices=1" "29 16 0.95 slices=16" "29 16 0.95 slices=32"; do
  timeout 200 python tools/rates.py $cfg reps=2 >> $O 2>> gpurun_out/knee.err
done
for ch in 28 29; do WD_SLICE_CHUNK_LOG2=$ch timeout 200 python tools/rates.py 29 16 0.5 slices=32 reps=2 | sed "s/}$/, \"chunk\": $ch}/" >> $O; done
