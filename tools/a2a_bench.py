"""NCCL all-to-all microbenchmark at the cascade's message sizes ("measure
[the exchange] against 900 GB/s per direction and against an all-to-all microbenchmark run
on the box — a timed ncclAlltoAll loop at the same message sizes").

    torchrun --nproc-per-node N tools/a2a_bench.py [--batch-log2 24] [--steps 20]

For a cascade batch of B items per GPU, every GPU sends ~B/N items to each peer: 8-B pairs
(insert), 4-B keys (query forward) and 8-B packed results (query reverse).  Each size is
timed with CUDA events around torch.distributed.all_to_all_single (NCCL) after a warm-up,
max over ranks.  Reported per GPU: algbw = bytes sent to the other ranks / time, and the
fraction of NVLink 5's 900 GB/s per direction.  Prints one JSON line per size (rank 0)."""
import argparse
import json
import os

import torch
import torch.distributed as dist


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--batch-log2", type=int, default=24)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    a = ap.parse_args()
    local = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    world, rank = dist.get_world_size(), dist.get_rank()
    B = 1 << a.batch_log2
    for name, isz in (("insert_pairs", 8), ("query_keys", 4), ("query_results", 8)):
        per_peer = (B // world) * isz
        x = torch.empty(per_peer * world, dtype=torch.uint8, device="cuda")
        y = torch.empty_like(x)
        for _ in range(a.warmup):
            dist.all_to_all_single(y, x)
        torch.cuda.synchronize()
        dist.barrier()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(a.steps):
            dist.all_to_all_single(y, x)
        e1.record()
        torch.cuda.synchronize()
        ms = torch.tensor([e0.elapsed_time(e1) / a.steps], dtype=torch.float64, device="cuda")
        dist.all_reduce(ms, op=dist.ReduceOp.MAX)
        ms = float(ms.item())
        sent = per_peer * (world - 1)
        gbs = sent / (ms * 1e-3) / 1e9
        if rank == 0:
            print(json.dumps({"tool": "a2a_bench", "n_gpus": world, "message": name,
                              "items_per_gpu": B, "bytes_per_peer": per_peer, "ms": ms,
                              "algbw_GBps_per_gpu": gbs, "frac_of_900GBps": gbs / 900.0}),
                  flush=True)
    dist.destroy_process_group()


if __name__ == "__main__":
    main()
