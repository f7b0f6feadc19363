#!/bin/bash
# GPU suite, headline bench, config 3/4/5 runners at N = 1 (refresh profiles/r02)
cd $GRAFT_REPO_ROOT
O=gpurun_out/r02i
mkdir -p $O
timeout 1200 python -m pytest tests -x -q -m gpu > $O/pytest.log 2>&1; echo "rc=$?" >> $O/pytest.log
timeout 600 python bench.py > $O/bench.json 2> $O/bench.err
for c in 3 4 5; do
  timeout 900 python bench.py --config $c --steps 3 --warmup 3 --no-cpu > $O/cfg$c.json 2> $O/cfg$c.err
done
