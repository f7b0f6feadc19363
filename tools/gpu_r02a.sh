#!/bin/bash
# round 2, session a: new full-size / sharded tests, the whole GPU suite, one bench line
cd $GRAFT_REPO_ROOT
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total --format=csv > gpurun_out/r02a_smi.txt
timeout 900 python -m pytest tests/test_gpu_gen.py tests/test_gpu_fullsize.py tests/test_gpu_loopback.py -x -q -m gpu --durations=15 > gpurun_out/r02a_pytest_new.log 2>&1
echo "rc_new=$?" >> gpurun_out/r02a_pytest_new.log
timeout 900 python -m pytest tests -x -q -m gpu > gpurun_out/r02a_pytest_all.log 2>&1
echo "rc_all=$?" >> gpurun_out/r02a_pytest_all.log
timeout 600 python bench.py > gpurun_out/r02a_bench.json 2> gpurun_out/r02a_bench.err
echo "rc_bench=$?" >> gpurun_out/r02a_bench.err
