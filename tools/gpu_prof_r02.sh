#!/bin/bash
# ncu full capture of one retrieve launch and one sliced-insert probe launch of the bench
# configuration, with source-level (CUDA line) instruction and stall attribution.
# usage: tools/gpu_prof_r02.sh TAG [extra bench args]
cd $GRAFT_REPO_ROOT
TAG=$1; shift
O=gpurun_out/prof_$TAG
mkdir -p $O
timeout 900 ncu --set full --clock-control none --import-source on -k regex:probe_ -s 62 -c 3 \
  -o $O/full python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu "$@" > $O/ncu.log 2>&1
ncu -i $O/full.ncu-rep --page raw --csv > $O/raw.csv 2>/dev/null
ncu -i $O/full.ncu-rep --page details --csv > $O/details.csv 2>/dev/null
ncu -i $O/full.ncu-rep --page source --csv --print-source cuda > $O/source_cuda.csv 2>/dev/null
ncu -i $O/full.ncu-rep --page source --csv --print-source sass > $O/source_sass.csv 2>/dev/null
rm -f $O/full.ncu-rep
ls -la $O
