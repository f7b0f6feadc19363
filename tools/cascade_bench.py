"""Loopback cascade measurement (m virtual shards on one GPU): insert / retrieve through
the full multi-GPU path (a6-a10) vs the single-shard path, same keys; for m > 1 both the fused
exchange (peer stores inside the kernels) and the staged copy-engine exchange, with the
per-phase decomposition; every query checked.  One JSON line per run."""
import math
import os
import sys

R = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, R)
import torch  # noqa: E402

import paper_conf_ipps_junger0s18_b200 as wd  # noqa: E402
import wdgen.gpu as gg  # noqa: E402


def run(n, m, batch, reps=3, G=4, exchange=0):
    keys, vals = gg.unique_keys(n, 3), gg.values(n, 4)
    vo = torch.empty(n, dtype=torch.int32, device="cuda")
    fo = torch.empty(n, dtype=torch.uint8, device="cuda")
    cap = int(math.ceil(n / 0.95))
    t = wd.Table(cap, 1, G) if m == 1 else wd.Table(cap, group_size=G, loopback_shards=m, batch=batch,
                                                      exchange=exchange)
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
    bad, first, found = gg.check_unique(keys, vo, fo, n, 3, 4)
    assert bad == 0 and found == n
    t.phase_times()
    t.set_option(wd.WD_OPT_PHASE_TIMING, 1)
    t.clear(s); t.insert(keys, vals, s)
    ph_i = {k: round(v[0], 3) for k, v in t.phase_times().items() if v[1]}
    t.retrieve(keys, vo, fo, s)
    ph_q = {k: round(v[0], 3) for k, v in t.phase_times().items() if v[1]}
    launches = t.launches
    t.close()
    return n / (sum(ti) / len(ti)) / 1e6, n / (sum(tq) / len(tq)) / 1e6, launches, ph_i, ph_q


if __name__ == "__main__":
    import json
    lg = int(sys.argv[1]) if len(sys.argv) > 1 else 26
    G = int(sys.argv[2]) if len(sys.argv) > 2 else 16
    n = 1 << lg
    for m in (1, 2, 4, 8):
        for x in ((0,) if m == 1 else (0, 1)):
            i, q, l, pi, pq = run(n, m, 1 << 24, G=G, exchange=x)
            print(json.dumps({"n_log2": lg, "G": G, "m": m, "exchange": ["fused", "copy engine"][x],
                              "insert_gops": i, "query_gops": q, "launches": l,
                              "insert_phases_ms": pi, "query_phases_ms": pq}), flush=True)
