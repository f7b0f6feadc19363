"""Small runs of every path for compute-sanitizer (memcheck / racecheck / synccheck)."""
import os, sys
R = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, R); sys.path.insert(0, os.path.join(R, "tests"))
import numpy as np, torch
import paper_conf_ipps_junger0s18_b200 as wd, wdgen, oracle
from wdtest import gpu_roundtrip, capacity_for
n = 20_000
keys, vals = wdgen.unique_keys(n, 1), wdgen.values(n, 2)
q = wdgen.interleaved_queries(n, 1)
cv, cf = oracle.expected_unique(q, n, 1, 2)
def check(gv, gf):
    assert np.array_equal(gf, cf) and np.array_equal(gv, cv)
for G, V in [(4, 1), (8, 4), (4, 4), (1, 1), (2, 2), (16, 8), (32, 8)]:  # (1,1), (2,2), (4,4): span S = 2
    with wd.Table(capacity_for(n, 0.9), 1, G) as t:
        t.set_option(wd.WD_OPT_SLOTS_PER_LANE, V)
        check(*gpu_roundtrip(t, keys, vals, q))
with wd.Table(capacity_for(n, 0.9), 1, 16) as t:   # slice-grouped bulk insert (forced)
    t.set_option(wd.WD_OPT_SLICES, 16)
    check(*gpu_roundtrip(t, keys, vals, q))
with wd.Table(capacity_for(n, 0.9), 1, 4) as t:
    t.set_option(wd.WD_OPT_SERIAL, 1)
    check(*gpu_roundtrip(t, keys, vals, q))
with wd.Table(capacity_for(n, 0.9), group_size=8, loopback_shards=3, batch=3000) as t:
    check(*gpu_roundtrip(t, keys, vals, q))
with wd.Table(capacity_for(n, 0.9), 1, 8, batch=3000) as t:
    check(*gpu_roundtrip(t, keys, vals, q, host=True))
# round 2 paths: V = 16 one-lane windows, the sliced insert with two chunks overlapped
# (forced small chunks are env-only, so two calls), the
# copy-engine exchange, the _sharded calls, erase through the staged reverse path
with wd.Table(capacity_for(n, 0.9), 1, 16) as t:
    t.set_option(wd.WD_OPT_SLOTS_PER_LANE, 16)
    check(*gpu_roundtrip(t, keys, vals, q))
for nbk, G in ((64, 16), (128, 4), (32, 8)):       # the 64- / 128-slot multisplit instances
    with wd.Table(capacity_for(n, 0.9), 1, G) as t:
        t.set_option(wd.WD_OPT_SLICES, nbk)
        check(*gpu_roundtrip(t, keys, vals, q))
with wd.Table(capacity_for(n, 0.9), 1, 8) as t:  # automatic rebuild after tombstones fill it
    t.set_option(wd.WD_OPT_AUTO_REBUILD, 1)
    t.insert(torch.from_numpy(keys.view(np.int32)).cuda(), torch.from_numpy(vals.view(np.int32)).cuda())
    t.erase(torch.from_numpy(keys[: n // 2].view(np.int32)).cuda())
    more = wdgen.unique_keys(n // 2, 1, start=n)
    t.insert(torch.from_numpy(more.view(np.int32)).cuda(), torch.from_numpy(wdgen.values(n // 2, 3).view(np.int32)).cuda())
    assert t.sync() == 0 and t.size() == n
with wd.Table(capacity_for(n, 0.9), group_size=8, loopback_shards=3, batch=3000, exchange=1) as t:
    check(*gpu_roundtrip(t, keys, vals, q))
    er = t.erase(torch.from_numpy(q[: n // 2].view(np.int32)).cuda())
    torch.cuda.synchronize()
    assert np.array_equal(er.cpu().numpy().astype(bool), cf[: n // 2].astype(bool))
with wd.Table(capacity_for(n, 0.9), group_size=4, loopback_shards=2, batch=4000) as t:
    import wdgen.gpu as gg
    half = n // 2
    ks = [gg.unique_keys(half, 1, start=r * half) for r in range(2)]
    vs = [gg.values(half, 2, start=r * half) for r in range(2)]
    t.insert_sharded(ks, vs)
    vo = [torch.empty(half, dtype=torch.int32, device="cuda") for _ in range(2)]
    fo = [torch.empty(half, dtype=torch.uint8, device="cuda") for _ in range(2)]
    t.retrieve_sharded(ks, vo, fo)
    torch.cuda.synchronize()
    for r in range(2):
        assert gg.check_unique(ks[r], vo[r], fo[r], n, 1, 2)[0] == 0
print("sanitize run ok")
