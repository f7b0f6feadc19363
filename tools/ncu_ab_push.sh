for l in pull16 push16; do
WD_LIBRARY=exp/lib$l.so timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sectors_op_write.sum,lts__t_sectors_op_read.sum --clock-control none --csv --log-file gpurun_out/casc_$l.csv python -c "
import sys; sys.path.insert(0,'tools'); sys.argv=['x']
import cascade_bench as cb
print(cb.run(1<<26, 2, 1<<24, reps=1, G=16))
" > /dev/null 2>&1
done
