#!/bin/bash
cd $GRAFT_REPO_ROOT
O=gpurun_out/r02e
mkdir -p $O
timeout 1200 python -m pytest tests -x -q -m gpu > $O/pytest.log 2>&1; echo "rc=$?" >> $O/pytest.log
timeout 600 python bench.py > $O/bench.json 2> $O/bench.err
for cfg in "29 16 0.5" "30 16 0.5" "28 16 0.95"; do timeout 200 python tools/rates.py $cfg reps=2 >> $O/rates.jsonl; done
