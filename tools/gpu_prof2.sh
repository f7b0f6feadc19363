# usage: bash tools/gpu_prof2.sh TAG REGEX [bench args]
TAG=$1; RX=$2; shift; shift
timeout 600 ncu --set full --clock-control none --import-source on -k regex:$RX -s 2 -c 2 -o gpurun_out/prof_$TAG python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu "$@" > gpurun_out/ncu_$TAG.log 2>&1
echo done
