#!/bin/bash
# deferred clear (fill overlapping the slice grouping): GPU suite, bench x2, smoke
cd $GRAFT_REPO_ROOT
O=gpurun_out/r02w
mkdir -p $O
timeout 1500 python -m pytest tests -x -q -m gpu > $O/pytest.log 2>&1; echo "rc=$?" >> $O/pytest.log
for i in 1 2; do timeout 600 python bench.py --no-cpu > $O/bench$i.json 2> $O/bench$i.err; done
timeout 300 python __graft_entry__.py > $O/smoke.log 2>&1; echo "rc=$?" >> $O/smoke.log
