#!/bin/bash
cd $GRAFT_REPO_ROOT
T=$1
timeout 600 python -m pytest tests/test_gpu_single.py tests/test_gpu_fullsize.py -x -q -m gpu > gpurun_out/${T}_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/${T}_pytest.log
bash tools/gpu_rates.sh ${T}_rates
