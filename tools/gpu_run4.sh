timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1
rm -f gpurun_out/kg.txt
for mode in 0 1; do for k in 0 4 8; do for g in 1 2 4 8; do
  timeout 120 python bench.py --steps 5 --warmup 2 --no-e2e --no-cpu --kif $k --group-size $g --probe-mode $mode 2>&1 | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('mode=$mode K=$k G=$g', round(d['insert_gops'],2), round(d['query_gops'],2), round(d['roofline']['frac'],3), round(d['roofline']['other']['frac'],3), d['clocks']['sm_mhz'])" >> gpurun_out/kg.txt 2>&1
done; done; done
echo done
