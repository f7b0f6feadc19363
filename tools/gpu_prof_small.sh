#!/bin/bash
# ncu of the config-1 insert / retrieve launches (2^20 keys, |g| = 4, L2-resident table)
cd $GRAFT_REPO_ROOT
TAG=$1; shift
O=gpurun_out/prof_$TAG
mkdir -p $O
timeout 900 ncu --set full --clock-control none --import-source on -k regex:probe_ -s 4 -c 2 \
  -o $O/full python tools/rates.py 20 4 q=inter reps=1 tail=0 "$@" > $O/ncu.log 2>&1
ncu -i $O/full.ncu-rep --page raw --csv > $O/raw.csv 2>/dev/null
ncu -i $O/full.ncu-rep --page details --csv > $O/details.csv 2>/dev/null
ncu -i $O/full.ncu-rep --page source --csv --print-source sass > $O/source_sass.csv 2>/dev/null
rm -f $O/full.ncu-rep
for mb in 74 148 296 592 0; do for k in 1 2 4; do
  WD_MAX_BLOCKS=$mb timeout 60 python tools/rates.py 20 4 q=inter reps=10 tail=0 k=$k | sed "s/}$/, \"max_blocks\": $mb}/" >> $O/grid.jsonl
done; done
