#!/bin/bash
cd $GRAFT_REPO_ROOT
T=$1
timeout 900 python -m pytest tests/test_gpu_single.py tests/test_gpu_loopback.py -x -q -m gpu -k "tail or split or serial or span or slice" > gpurun_out/${T}_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/${T}_pytest.log
: > gpurun_out/${T}.jsonl
for tl in -1 0; do
  for cfg in "20 4 q=inter" "20 8 q=inter" "20 16 q=inter" "22 4" "22 16" "24 4"; do
    timeout 120 python tools/rates.py $cfg tail=$tl reps=10 >> gpurun_out/${T}.jsonl 2>> gpurun_out/${T}.err
  done
done
make -s tools/randbench 2>/dev/null || nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o tools/randbench tools/randbench.cu
./tools/randbench 0.0088 0.035 > gpurun_out/${T}_randbench_l2.txt 2>&1
