# A/B of two library builds on the loopback cascade: per-kernel times + DRAM bytes (ncu)
# and call rates (cascade_bench).  usage: bash tools/ncu_ab_ms.sh libA libB tag
for l in $1 $2; do
  t=$(basename $l .so)
  WD_LIBRARY=$l timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/ms_${3}_$t.csv python -c "
import sys; sys.path.insert(0,'tools'); sys.argv=['x']
import cascade_bench as cb
print(cb.run(1<<26, 8, 1<<24, reps=1, G=16))
" > /dev/null 2>&1
done
for r in 1 2; do for l in $1 $2; do echo "== $l"; WD_LIBRARY=$l python tools/cascade_bench.py 28 16; done; done > gpurun_out/ms_${3}_rates.txt 2>&1
