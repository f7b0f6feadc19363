#!/bin/bash
# session 3: N = 2 same-device dry runs of configs 2-5 (fused / copy-engine exchange) and the
# loopback cascade bench on the new multisplit
cd $GRAFT_REPO_ROOT
O=gpurun_out/r02u
mkdir -p $O
TR="python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port"
P=29611
for x in 0 1; do
  for c in 2 3 4 5; do
    case $c in 2) n=24;; 3) n=26;; 4) n=25;; 5) n=24;; esac
    P=$((P+1))
    timeout 300 $TR $P bench.py --gpus 2 --same-device --config $c --n-log2 $n --exchange $x --steps 3 --warmup 3 --no-e2e --no-cpu --batch-log2 22 > $O/dry_c${c}_x$x.json 2> $O/dry_c${c}_x$x.err; echo "rc=$?" >> $O/dry_c${c}_x$x.err
  done
done
timeout 600 python tools/cascade_bench.py > $O/cascade.jsonl 2> $O/cascade.err
