#!/bin/bash
# final-library evidence: GPU suite, launch list + full captures, bench, config-2 sweep
cd $GRAFT_REPO_ROOT
O=gpurun_out/r02h
mkdir -p $O
timeout 1200 python -m pytest tests -x -q -m gpu > $O/pytest.log 2>&1; echo "rc=$?" >> $O/pytest.log
bash tools/gpu_evidence_r02.sh r02h
timeout 2000 python bench.py --sweep --no-cpu --no-e2e --steps 3 > $O/sweep.jsonl 2> $O/sweep.err
