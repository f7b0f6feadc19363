#!/bin/bash
# session-3 evidence: ncu launch list of the bench (per-launch time + DRAM bytes), full
# captures of the multisplit (segment mode) and both probe kernels, configs 3/4/5 at N = 1
cd $GRAFT_REPO_ROOT
O=gpurun_out/r02p
mkdir -p $O
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
  -c 200 --csv --log-file $O/launches.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu > $O/ncu_list.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:multisplit_kernel -c 1 \
  -o $O/full_ms python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu > $O/ncu_full_ms.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:probe_ -s 31 -c 2 \
  -o $O/full_probe python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu > $O/ncu_full_probe.log 2>&1
for f in full_ms full_probe; do
  ncu -i $O/$f.ncu-rep --page raw --csv > $O/${f}_raw.csv 2>/dev/null
  ncu -i $O/$f.ncu-rep --page details --csv > $O/${f}_details.csv 2>/dev/null
done
rm -f $O/*.ncu-rep
for c in 3 4 5; do
  timeout 900 python bench.py --config $c --steps 3 --warmup 3 --no-cpu > $O/cfg$c.json 2> $O/cfg$c.err
done
