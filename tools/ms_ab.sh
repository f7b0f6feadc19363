# multisplit / unpermute kernel times for library builds given as arguments (ncu launch list)
for l in "$@"; do
  t=$(basename $l .so)
  WD_LIBRARY=$l ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/msab_$t.csv python tools/ms_prof.py 27 8 24 > /dev/null 2>&1
done
