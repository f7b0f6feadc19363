#!/bin/bash
# round-2 evidence of the bench configuration: ncu launch list with DRAM bytes per launch
# (-> profiles/traffic.json), a full capture of the two probe kernels, the GPU suite, bench
cd $GRAFT_REPO_ROOT
T=${1:-r02f}
O=gpurun_out/$T
mkdir -p $O
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
  -c 200 --csv --log-file $O/launches.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu > $O/ncu_list.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:probe_ -s 31 -c 2 \
  -o $O/full python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu > $O/ncu_full.log 2>&1
ncu -i $O/full.ncu-rep --page raw --csv > $O/raw.csv 2>/dev/null
ncu -i $O/full.ncu-rep --page details --csv > $O/details.csv 2>/dev/null
ncu -i $O/full.ncu-rep --page source --csv --print-source sass > $O/source_sass.csv 2>/dev/null
rm -f $O/full.ncu-rep
timeout 600 python bench.py > $O/bench.json 2> $O/bench.err
