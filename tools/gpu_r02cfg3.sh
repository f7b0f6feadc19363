#!/bin/bash
# config 3 at N = 1: the library at bbdefe8 (before the 4-block insert and the insert |g|
# option) vs the current one, alternating, on the same box
cd $GRAFT_REPO_ROOT
O=gpurun_out/r02cfg3b
mkdir -p $O
for rep in 1 2; do
  timeout 900 python bench.py --config 3 --steps 3 --warmup 3 --no-cpu > $O/cur_$rep.json 2> $O/cur_$rep.err
  WD_LIBRARY=build/ab/lib_bbdefe8.so timeout 900 python bench.py --config 3 --steps 3 --warmup 3 --no-cpu > $O/old_$rep.json 2> $O/old_$rep.err
done
