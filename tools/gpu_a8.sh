#!/bin/bash
# region-alignment change: GPU tests, A/B against the 4-slot build, L2 fetch limit A/B, bench
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/a8_tests.txt 2>&1; echo "tests rc=$?" >> gpurun_out/a8_tests.txt
bash tools/ab_lib.sh abso/libwarpdrive_seq.so abso/libwarpdrive_a8.so cfg 28 8:4:2 8:4:4 8:0:0 4:0:0 16:0:0 8:1:4 > gpurun_out/a8_ab.txt 2>&1
for fb in 32 64 128; do echo "== WD_L2_FETCH_BYTES=$fb"; WD_L2_FETCH_BYTES=$fb python tools/kbench.py cfg 28 8:0:0 4:0:0 16:0:0; done > gpurun_out/a8_fetch.txt 2>&1
python bench.py > gpurun_out/a8_bench.txt 2>&1
