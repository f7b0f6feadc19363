"""Kernel-level rate sweep (measurement tool): insert / retrieve G ops/s for table sizes
from L2-resident (config 1) to HBM-sized (config 2), per probe mode and |g|."""
import math
import os
import sys

R = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, R)
import torch  # noqa: E402

import paper_conf_ipps_junger0s18_b200 as wd  # noqa: E402
import wdgen.gpu as gg  # noqa: E402


def rate(n, G, mode, alpha=0.95, kif=0, reps=5, spl=0):
    keys, vals = gg.unique_keys(n, 1), gg.values(n, 2)
    vo = torch.empty(n, dtype=torch.int32, device="cuda")
    fo = torch.empty(n, dtype=torch.uint8, device="cuda")
    t = wd.Table(int(math.ceil(n / alpha)), 1, G)
    t.set_option(wd.WD_OPT_PROBE_MODE, mode)
    if kif:
        t.set_option(wd.WD_OPT_KEYS_IN_FLIGHT, kif)
    if spl:
        t.set_option(wd.WD_OPT_SLOTS_PER_LANE, spl)
    s = torch.cuda.current_stream()
    ti, tq = [], []
    for r in range(reps + 1):
        a, b, c = (torch.cuda.Event(enable_timing=True) for _ in range(3))
        t.clear(s)
        a.record(s); t.insert(keys, vals, s); b.record(s); t.retrieve(keys, vo, fo, s); c.record(s)
        torch.cuda.synchronize()
        if r:
            ti.append(a.elapsed_time(b)); tq.append(b.elapsed_time(c))
    assert t.sync() == 0 and t.size() == n
    t.close()
    return n / (sum(ti) / len(ti)) / 1e6, n / (sum(tq) / len(tq)) / 1e6


if __name__ == "__main__" and (len(sys.argv) < 2 or sys.argv[1] not in ("noout", "split", "cfg")):
    if len(sys.argv) > 1 and sys.argv[1] == "k":
        lg = int(sys.argv[2]) if len(sys.argv) > 2 else 28
        for G, m, ks in [(4, 1, (2, 4, 8)), (4, 2, (1, 2, 4, 8)), (8, 2, (1, 2, 4)),
                         (2, 2, (2, 4, 8)), (8, 1, (2, 4, 8)), (1, 2, (2, 4, 8))]:
            for k in ks:
                i, q = rate(1 << lg, G, m, kif=k)
                print(f"n=2^{lg} G={G} mode={m} K={k}: insert {i:6.2f} G/s  query {q:6.2f} G/s",
                      flush=True)
        sys.exit(0)
    cfgs = [(G, m) for m in (1, 2) for G in (2, 4, 8)]
    for lg in (20, 22, 24, 26, 28):
        for G, m in cfgs:
            i, q = rate(1 << lg, G, m)
            print(f"n=2^{lg} G={G} mode={m}: insert {i:6.2f} G/s  query {q:6.2f} G/s", flush=True)


def query_no_out(n, G, mode, kif=0, alpha=0.95, reps=5):
    """retrieve with vals_out = found_out = NULL: probing only, no output stores"""
    keys, vals = gg.unique_keys(n, 1), gg.values(n, 2)
    t = wd.Table(int(math.ceil(n / alpha)), 1, G)
    t.set_option(wd.WD_OPT_PROBE_MODE, mode)
    if kif:
        t.set_option(wd.WD_OPT_KEYS_IN_FLIGHT, kif)
    s = torch.cuda.current_stream()
    t.insert(keys, vals, s)
    ts = []
    for r in range(reps + 1):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(s)
        wd.wd_retrieve(t.handle, keys.data_ptr(), None, None, n, s.cuda_stream)
        b.record(s)
        torch.cuda.synchronize()
        if r:
            ts.append(a.elapsed_time(b))
    t.close()
    return n / (sum(ts) / len(ts)) / 1e6


if __name__ == "__main__" and len(sys.argv) > 1 and sys.argv[1] == "noout":
    for G, m, k in [(4, 1, 8), (4, 2, 4), (4, 2, 1), (8, 1, 4), (8, 2, 2), (1, 2, 8)]:
        print(f"G={G} mode={m} K={k}: query without outputs {query_no_out(1 << 28, G, m, k):6.2f} G/s; "
              f"with: {rate(1 << 28, G, m, kif=k)[1]:6.2f} G/s", flush=True)


if __name__ == "__main__" and len(sys.argv) > 1 and sys.argv[1] == "split":
    lg = int(sys.argv[2]) if len(sys.argv) > 2 else 28
    for G, V, ks in [(4, 1, (4, 8)), (4, 2, (4, 8)), (4, 4, (2, 4)), (8, 1, (4, 8)), (8, 2, (4, 8)),
                     (8, 4, (2, 4)), (8, 8, (2,)), (2, 1, (4, 8)), (2, 2, (4, 8)), (16, 2, (4, 8)),
                     (16, 4, (2, 4))]:
        for k in ks:
            i, q = rate(1 << lg, G, 0, kif=k, spl=V)
            print(f"n=2^{lg} G={G} V={V} K={k}: insert {i:6.2f} G/s  query {q:6.2f} G/s", flush=True)


if __name__ == "__main__" and len(sys.argv) > 1 and sys.argv[1] == "cfg":
    # kbench.py cfg <lg> G:V:K ...   (V = 0: auto, K = 0: auto)
    lg = int(sys.argv[2])
    for c in sys.argv[3:]:
        G, V, k = (int(x) for x in c.split(":"))
        i, q = rate(1 << lg, G, 0, kif=k, spl=V)
        print(f"n=2^{lg} G={G} V={V} K={k}: insert {i:6.2f} G/s  query {q:6.2f} G/s", flush=True)
