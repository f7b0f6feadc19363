"""Loopback cascade measurement (m virtual shards on one GPU): insert / retrieve through
the full multi-GPU path (a6-a10) vs the single-shard path, same keys.  Per-kernel times
come from an ncu launch list of this script (tools/gpu_cascade.sh)."""
import math
import os
import sys

R = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, R)
import torch  # noqa: E402

import paper_conf_ipps_junger0s18_b200 as wd  # noqa: E402
import wdgen.gpu as gg  # noqa: E402


def run(n, m, batch, reps=3, G=4):
    keys, vals = gg.unique_keys(n, 3), gg.values(n, 4)
    vo = torch.empty(n, dtype=torch.int32, device="cuda")
    fo = torch.empty(n, dtype=torch.uint8, device="cuda")
    cap = int(math.ceil(n / 0.95))
    t = wd.Table(cap, 1, G) if m == 1 else wd.Table(cap, group_size=G, loopback_shards=m, batch=batch)
    s = torch.cuda.current_stream()
    ti, tq = [], []
    for r in range(reps + 1):
        a, b, c = (torch.cuda.Event(enable_timing=True) for _ in range(3))
        t.clear(s)
        a.record(s); t.insert(keys, vals, s); b.record(s); t.retrieve(keys, vo, fo, s); c.record(s)
        torch.cuda.synchronize()
        if r:
            ti.append(a.elapsed_time(b)); tq.append(b.elapsed_time(c))
    assert t.sync() == 0 and t.size() == n, (t.sync(), t.size())
    idx = torch.randint(0, n, (1 << 16,), device="cuda")
    assert bool((fo[idx] == 1).all()) and bool((vo[idx] == vals[idx]).all())
    launches = t.launches
    t.close()
    return n / (sum(ti) / len(ti)) / 1e6, n / (sum(tq) / len(tq)) / 1e6, launches


if __name__ == "__main__":
    lg = int(sys.argv[1]) if len(sys.argv) > 1 else 26
    G = int(sys.argv[2]) if len(sys.argv) > 2 else 16
    n = 1 << lg
    for m in (1, 2, 4, 8):
        i, q, l = run(n, m, 1 << 24, G=G)
        print(f"n=2^{lg} |g|={G} loopback m={m} batch=2^24: insert {i:6.2f} G/s  query {q:6.2f} G/s  "
              f"(launches {l})", flush=True)
