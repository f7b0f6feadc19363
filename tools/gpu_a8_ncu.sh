#!/bin/bash
mkdir -p gpurun_out
for tag in seq a8; do
  WD_LIBRARY=abso/libwarpdrive_$tag.so timeout 900 ncu --set full --clock-control none -k regex:probe_kernel -s 2 -c 2 \
      -o /tmp/ncu_align_$tag -f python tools/kbench.py cfg 28 8:4:2 > gpurun_out/ncu_align_$tag.log 2>&1
  ncu -i /tmp/ncu_align_$tag.ncu-rep --page raw --csv > gpurun_out/ncu_align_$tag.csv 2>&1
done
ls -la /tmp/ncu_align_* gpurun_out/ >> gpurun_out/ncu_align_seq.log
