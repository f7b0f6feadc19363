"""Capacity sweep (P:219 / SURVEY 8(f) #4: is there a large-table knee on B200?): insert and
retrieve rates at alpha 0.95 from 2^24 to 2^32-1 unique keys (config 3 at m = 1: 36 GB table),
each checked on a sample against the closed form."""
import math, os, sys
R = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, R)
import numpy as np, torch
import paper_conf_ipps_junger0s18_b200 as wd
import wdgen.gpu as gg
import oracle

G = int(sys.argv[1]) if len(sys.argv) > 1 else 8
for lg in (24, 26, 28, 29, 30, 31, 32):
    n = (1 << lg) if lg < 32 else (1 << 32) - 1
    keys = gg.unique_keys(n, 11)
    vals = gg.values(n, 12)
    t = wd.Table(int(math.ceil(n / 0.95)), 1, G)
    s = torch.cuda.current_stream()
    vo = torch.empty(n, dtype=torch.int32, device="cuda")
    fo = torch.empty(n, dtype=torch.uint8, device="cuda")
    ti, tq = [], []
    for r in range(3 if lg < 31 else 2):
        a, b, c = (torch.cuda.Event(enable_timing=True) for _ in range(3))
        t.clear(s); a.record(s); t.insert(keys, vals, s); b.record(s); t.retrieve(keys, vo, fo, s); c.record(s)
        torch.cuda.synchronize()
        if r: ti.append(a.elapsed_time(b)); tq.append(b.elapsed_time(c))
    assert t.sync() == 0 and t.size() == n
    idx = torch.randint(0, n, (1 << 20,), device="cuda", dtype=torch.int64)
    qs = keys[idx].cpu().numpy().view(np.uint32)
    ev, ef = oracle.expected_unique(qs, n, 11, 12)
    ok = np.array_equal(fo[idx].cpu().numpy(), ef) and np.array_equal(vo[idx].cpu().numpy().view(np.uint32), ev)
    print(f"n={n} ({t.capacity()*8/1e9:.2f} GB table) G={G}: insert {n/(sum(ti)/len(ti))/1e6:6.2f} G/s  "
          f"query {n/(sum(tq)/len(tq))/1e6:6.2f} G/s  sample-parity {'ok' if ok else 'FAIL'}", flush=True)
    del keys, vals, vo, fo, t
    torch.cuda.empty_cache()
