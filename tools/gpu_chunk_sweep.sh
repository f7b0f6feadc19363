#!/bin/bash
# sliced insert with overlapped grouping: chunk size sweep (2^28 pairs, |g| = 16), + tests
cd $GRAFT_REPO_ROOT
O=gpurun_out/${1:-chsweep}.jsonl
: > $O
for ch in 25 26 27 28; do
  WD_SLICE_CHUNK_LOG2=$ch timeout 120 python tools/rates.py 28 16 reps=4 | sed "s/}$/, \"chunk_log2\": $ch}/" >> $O
done
timeout 600 python -m pytest tests/test_gpu_single.py tests/test_gpu_fullsize.py -x -q -m gpu > gpurun_out/${1:-chsweep}_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/${1:-chsweep}_pytest.log
