#!/bin/bash
# final session-3 evidence on the committed library: GPU suite, bench (default contract),
# ncu launch list of the same command, --set full capture of the probe + multisplit kernels
cd $GRAFT_REPO_ROOT
O=gpurun_out/r02x
mkdir -p $O
timeout 1500 python -m pytest tests -x -q -m gpu > $O/pytest.log 2>&1; echo "rc=$?" >> $O/pytest.log
timeout 600 python bench.py > $O/bench.json 2> $O/bench.err
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
  -c 200 --csv --log-file $O/launches.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu > $O/ncu_list.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"probe_|multisplit" -s 31 -c 3 \
  -o $O/full python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu > $O/ncu_full.log 2>&1
ncu -i $O/full.ncu-rep --page details --csv > $O/full_details.csv 2>/dev/null
ncu -i $O/full.ncu-rep --page raw --csv > $O/full_raw.csv 2>/dev/null
rm -f $O/full.ncu-rep
