#!/bin/bash
# PDL A/B for the slice probe launches (trigger when a warp's input is exhausted)
cd $GRAFT_REPO_ROOT
O=gpurun_out/r02m
mkdir -p $O
for i in 1 2; do
  timeout 600 python bench.py --no-cpu --no-e2e > $O/bench_pdl$i.json 2> $O/bench_pdl$i.err
  WD_NO_PDL=1 timeout 600 python bench.py --no-cpu --no-e2e > $O/bench_nopdl$i.json 2> $O/bench_nopdl$i.err
done
timeout 1200 python -m pytest tests/test_gpu_fullsize.py -x -q -m gpu -k bench_configuration > $O/pytest.log 2>&1; echo "rc=$?" >> $O/pytest.log
