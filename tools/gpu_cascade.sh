python tools/cascade_bench.py 28 16 > gpurun_out/cascade.txt 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/cascade_launches.csv python -c "
import sys; sys.path.insert(0,'tools'); sys.argv=['x']
import cascade_bench as cb
print(cb.run(1<<26, 4, 1<<24, reps=1, G=16))
" > /dev/null 2>&1
echo done
