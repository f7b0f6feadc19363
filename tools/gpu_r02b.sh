#!/bin/bash
# round 2, session b: exchange modes (fused / copy engine) in loopback and rank mode
cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests/test_gpu_loopback.py tests/test_gpu_rank.py tests/test_gpu_erase.py -x -q -m gpu > gpurun_out/r02b_pytest.log 2>&1
echo "rc=$?" >> gpurun_out/r02b_pytest.log
