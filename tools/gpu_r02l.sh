#!/bin/bash
# round-2 session 3: new multisplit (segment mode) — ms_bench, GPU suite, headline bench
cd $GRAFT_REPO_ROOT
O=gpurun_out/r02l
mkdir -p $O
#timeout 300 tools/ms_bench 28 10 > $O/ms_bench.txt 2>&1
timeout 1500 python -m pytest tests -x -q -m gpu > $O/pytest.log 2>&1; echo "rc=$?" >> $O/pytest.log
timeout 600 python bench.py > $O/bench.json 2> $O/bench.err
