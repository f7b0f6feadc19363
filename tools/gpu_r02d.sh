#!/bin/bash
# probe accounting under concurrency, capacity sweep at fixed load, random-access ceilings by size
cd $GRAFT_REPO_ROOT
O=gpurun_out/r02d
mkdir -p $O
timeout 900 python tools/probe_counts.py 28 > $O/probe_counts.jsonl 2> $O/probe_counts.err
timeout 900 python tools/size_sweep2.py 16 0.5 > $O/size_sweep2.jsonl 2> $O/size_sweep2.err
./tools/randbench 2.26 9 36 72 > $O/randbench_sizes.txt 2>&1
