#!/bin/bash
cd $GRAFT_REPO_ROOT
for lib in paper_conf_ipps_junger0s18_b200/libwarpdrive.so exp/ms2/libwarpdrive.so exp/ms4/libwarpdrive.so; do
  WD_LIBRARY=$lib timeout 120 python tools/rates.py 28 16 reps=3 | sed "s|}$|, \"lib\": \"$lib\"}|"
done > gpurun_out/ms_ab.jsonl 2>&1
