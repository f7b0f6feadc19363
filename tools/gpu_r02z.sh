#!/bin/bash
# auto insert + query |g|: GPU suite, headline bench, config-2 / config-1 / config-4 sweep
cd $GRAFT_REPO_ROOT
O=gpurun_out/r02z
mkdir -p $O
timeout 1500 python -m pytest tests -x -q -m gpu > $O/pytest.log 2>&1; echo "rc=$?" >> $O/pytest.log
timeout 600 python bench.py > $O/bench.json 2> $O/bench.err
timeout 1500 python bench.py --sweep --no-cpu --no-e2e > $O/sweep.jsonl 2> $O/sweep.err
