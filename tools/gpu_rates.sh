#!/bin/bash
# rate sweep: lean vs classic kernel on L2-resident and HBM tables (tools/rates.py)
cd $GRAFT_REPO_ROOT
T=${1:-rates}
O=gpurun_out/$T.jsonl
: > $O
for k in lean classic; do
  for cfg in "20 4" "22 8" "22 16" "24 16" "28 16" "28 16 slices=1" "28 8" "28 4"; do
    WD_PROBE_KERNEL=$k timeout 120 python tools/rates.py $cfg >> $O 2>> gpurun_out/$T.err
  done
done
