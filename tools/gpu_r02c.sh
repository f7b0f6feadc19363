#!/bin/bash
# round 2, session c: bench runners for BASELINE configs 3/4/5 at N = 1 (full size) and the
# N = 2 same-device dry runs (rank mode, gloo control plane) of every config and exchange
cd $GRAFT_REPO_ROOT
O=gpurun_out/r02c
mkdir -p $O
free -g > $O/host_mem.txt
for c in 3 4 5; do
  timeout 600 python bench.py --config $c --steps 3 --warmup 3 --no-cpu > $O/cfg$c.json 2> $O/cfg$c.err; echo "rc=$?" >> $O/cfg$c.err
done
TR="python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port"
P=29611
for x in 0 1; do
  for c in 2 3 4 5; do
    case $c in 2) n=24;; 3) n=26;; 4) n=25;; 5) n=24;; esac
    P=$((P+1))
    timeout 300 $TR $P bench.py --gpus 2 --same-device --config $c --n-log2 $n --exchange $x --steps 3 --warmup 3 --no-e2e --no-cpu --batch-log2 22 > $O/dry_c${c}_x$x.json 2> $O/dry_c${c}_x$x.err; echo "rc=$?" >> $O/dry_c${c}_x$x.err
  done
done
timeout 200 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 --master-port 29700 tools/a2a_bench.py --steps 5 > $O/a2a_w1.json 2> $O/a2a_w1.err
