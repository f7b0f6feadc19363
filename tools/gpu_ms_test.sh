#!/bin/bash
cd $GRAFT_REPO_ROOT
T=$1
for ch in 27 28; do WD_SLICE_CHUNK_LOG2=$ch timeout 120 python tools/rates.py 28 16 reps=3 | sed "s/}$/, \"chunk_log2\": $ch}/"; done > gpurun_out/${T}.jsonl 2>&1
timeout 900 python -m pytest tests/test_gpu_loopback.py tests/test_gpu_rank.py tests/test_gpu_single.py -x -q -m gpu > gpurun_out/${T}_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/${T}_pytest.log
