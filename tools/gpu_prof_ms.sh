#!/bin/bash
# ncu full capture of one grouping multisplit launch (bench configuration) + bench line
cd $GRAFT_REPO_ROOT
TAG=$1; shift
O=gpurun_out/prof_$TAG
mkdir -p $O
timeout 600 python bench.py --no-cpu > $O/bench.json 2> $O/bench.err
timeout 900 ncu --set full --clock-control none --import-source on -k regex:multisplit -s 1 -c 1 \
  -o $O/full python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu > $O/ncu.log 2>&1
ncu -i $O/full.ncu-rep --page raw --csv > $O/raw.csv 2>/dev/null
ncu -i $O/full.ncu-rep --page details --csv > $O/details.csv 2>/dev/null
ncu -i $O/full.ncu-rep --page source --csv --print-source sass > $O/source_sass.csv 2>/dev/null
rm -f $O/full.ncu-rep
