#!/bin/bash
# final: GPU suite, headline bench, configs 3/4/5 at N = 1
cd $GRAFT_REPO_ROOT
O=gpurun_out/r02fin2
mkdir -p $O
timeout 1500 python -m pytest tests -x -q -m gpu > $O/pytest.log 2>&1; echo "rc=$?" >> $O/pytest.log
timeout 600 python bench.py > $O/bench.json 2> $O/bench.err
for c in 3 4 5; do
  timeout 900 python bench.py --config $c --steps 3 --warmup 3 --no-cpu > $O/cfg$c.json 2> $O/cfg$c.err
done
