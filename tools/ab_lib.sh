#!/bin/bash
# A/B of two builds of libwarpdrive.so: tools/ab_lib.sh <lib_a> <lib_b> [kbench args...]
a=$1; b=$2; shift 2
for r in 1 2; do
  for l in "$a" "$b"; do
    echo "== $l (round $r)"; WD_LIBRARY=$l python tools/kbench.py "$@"
  done
done
