#!/bin/bash
# cursor-mode multisplit (the cascade): tile size x occupancy variants (tools/ms_bench.cu)
mkdir -p gpurun_out
for b in tools/ms_bench_c*; do echo "### $b"; timeout 200 $b 28 10 | grep -E "cascade_m|ok"; done > gpurun_out/ms_cursor.txt 2>&1
