#!/bin/bash
# lean probe kernel: GPU suite, then bench A/B against the round-1 kernel (WD_PROBE_KERNEL=classic)
cd $GRAFT_REPO_ROOT
T=${1:-lean}
O=gpurun_out/$T
mkdir -p $O
timeout 900 python -m pytest tests -x -q -m gpu > $O/pytest.log 2>&1; echo "rc=$?" >> $O/pytest.log
for k in lean classic lean classic; do
  WD_PROBE_KERNEL=$k timeout 300 python bench.py --no-e2e --no-cpu >> $O/bench_$k.json 2>> $O/bench_$k.err
done
