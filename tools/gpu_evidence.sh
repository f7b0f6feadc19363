# full evidence run: tests, smoke, ncu launch list (time + DRAM bytes per launch), ncu full capture
# of one retrieve launch and one slice launch of the insert (-s 64: 64 slice launches + 1 retrieve per step),
# DRAM traffic per call (profiles/traffic.json, the roofline`s `traffic`), then the bench line
TAG=${1:-r01}
G=${G:-16}
timeout 900 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu_$TAG.log 2>&1
timeout 300 python __graft_entry__.py > gpurun_out/smoke_$TAG.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_$TAG.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu > /dev/null 2>&1
python tools/traffic_per_call.py gpurun_out/launches_$TAG.csv $G > gpurun_out/traffic_call_$TAG.log 2>&1
# the report can exceed gpurun's 64 MiB return limit: keep it in /tmp, bring back CSV pages
timeout 900 ncu --set full --clock-control none --import-source on -k regex:probe -s 64 -c 2 -o /tmp/full_$TAG python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu > gpurun_out/ncu_$TAG.log 2>&1
ncu -i /tmp/full_$TAG.ncu-rep --page raw --csv > gpurun_out/full_${TAG}_raw.csv 2>/dev/null
ncu -i /tmp/full_$TAG.ncu-rep --page source --csv --print-source sass > gpurun_out/full_${TAG}_sass.csv 2>/dev/null
ncu -i /tmp/full_$TAG.ncu-rep --page details --csv > gpurun_out/full_${TAG}_details.csv 2>/dev/null
cp profiles/traffic.json gpurun_out/traffic_$TAG.json
timeout 600 python bench.py > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err
echo done
