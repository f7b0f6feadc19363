timeout 1800 python bench.py --steps 3 --warmup 3 --no-e2e --no-cpu --sweep > gpurun_out/sweep.jsonl 2> gpurun_out/sweep.err
echo done
