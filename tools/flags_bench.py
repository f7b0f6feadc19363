"""A/B of the kernel variants (WD_OPT_KERNEL_FLAGS) on unique (2^28) and Zipf (2^25 draws)."""
import math, os, sys
R = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, R)
import torch
import paper_conf_ipps_junger0s18_b200 as wd
import wdgen.gpu as gg


def rates(keys, vals, cap, G, mode, flags, reps=3):
    n = keys.numel()
    vo = torch.empty(n, dtype=torch.int32, device="cuda")
    fo = torch.empty(n, dtype=torch.uint8, device="cuda")
    t = wd.Table(cap, 1, G)
    t.set_option(wd.WD_OPT_PROBE_MODE, mode)
    t.set_option(wd.WD_OPT_KERNEL_FLAGS, flags)
    s = torch.cuda.current_stream()
    ti, tq = [], []
    for r in range(reps + 1):
        a, b, c = (torch.cuda.Event(enable_timing=True) for _ in range(3))
        t.clear(s); a.record(s); t.insert(keys, vals, s); b.record(s); t.retrieve(keys, vo, fo, s); c.record(s)
        torch.cuda.synchronize()
        if r:
            ti.append(a.elapsed_time(b)); tq.append(b.elapsed_time(c))
    assert t.sync() == 0 and bool((fo == 1).all())
    t.close()
    return n / (sum(ti) / len(ti)) / 1e6, n / (sum(tq) / len(tq)) / 1e6


nu = 1 << 28
uk, uv = gg.unique_keys(nu, 1), gg.values(nu, 2)
for mode, G in [(1, 4), (1, 8), (2, 4)]:
    for flags in (0, 1, 2, 3):
        i, q = rates(uk, uv, int(math.ceil(nu / 0.95)), G, mode, flags)
        print(f"unique 2^28 mode={mode} G={G} flags={flags}: insert {i:6.2f} query {q:6.2f}", flush=True)
del uk, uv
nz = 1 << 25
zk, zv = gg.zipf_keys(nz, 2**32 - 1, 5), gg.values(nz, 6)
distinct = int(torch.unique(zk).numel())
for mode, G in [(1, 1), (1, 4), (2, 4)]:
    for flags in (0, 1, 2, 3):
        i, q = rates(zk, zv, int(math.ceil(distinct / 0.95)), G, mode, flags)
        print(f"zipf 2^25 mode={mode} G={G} flags={flags}: insert {i:6.3f} query {q:6.2f}", flush=True)
