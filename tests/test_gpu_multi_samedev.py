"""The single-process multi-GPU mode (wd_create with n_gpus > 1: per-shard streams, host
input split into portions; the device-sided _sharded calls, P:175 / P:199; the
device-pointer rules) on ONE GPU: the library's test hook WD_MULTI_SAME_DEVICE puts every
shard on the current device.  The same checks as tests/test_gpu_multi.py (which needs >= 2
physical devices); every query against the generator's closed form.  NCCL (exchange 2)
needs distinct devices and is left to test_gpu_multi.py."""
import math

import numpy as np
import pytest

pytestmark = pytest.mark.gpu

KS, VS = 511, 512


@pytest.fixture
def samedev(monkeypatch):
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    monkeypatch.setenv("WD_MULTI_SAME_DEVICE", "1")
    torch.cuda.set_device(0)


@pytest.mark.parametrize("m,G,exchange", [(2, 4, 0), (3, 16, 0), (4, 16, 1), (8, 8, 0)])
def test_multi_mode_host_input(samedev, m, G, exchange):
    import torch
    import oracle
    import paper_conf_ipps_junger0s18_b200 as wd
    import wdgen
    n = 700_001
    keys, vals = wdgen.unique_keys(n, KS), wdgen.values(n, VS)
    q = wdgen.interleaved_queries(n, KS)
    with wd.Table(int(math.ceil(n / 0.9)), m, G, exchange=exchange) as t:
        assert t.get_option(wd.WD_OPT_N_SHARDS) == m
        t.set_option(wd.WD_OPT_BATCH, 1 << 17)           # several batches per shard
        kk = torch.from_numpy(keys.view(np.int32)).pin_memory()
        vv = torch.from_numpy(vals.view(np.int32)).pin_memory()
        t.insert(kk, vv)
        qq = torch.from_numpy(q.view(np.int32)).pin_memory()
        ov = torch.empty(q.size, dtype=torch.int32).pin_memory()
        of = torch.empty(q.size, dtype=torch.uint8).pin_memory()
        t.retrieve(qq, ov, of)
        torch.cuda.synchronize()
        assert t.sync() == 0, wd._lib.wd_last_error_message()
        assert t.size() == n
        seed = t.get_option(wd.WD_OPT_PART_SEED)
        for d in range(m):                                 # shard d holds p(k) = d
            sl = t.dump(d)
            k = (sl & np.uint64(0xFFFFFFFF)).astype(np.uint32)
            k = k[k != np.uint32(0xFFFFFFFF)]
            assert np.all(oracle.partition(k, m, seed) == d)
    cv, cf = oracle.expected_unique(q, n, KS, VS)
    assert np.array_equal(of.numpy(), cf) and np.array_equal(ov.numpy().view(np.uint32), cv)


@pytest.mark.parametrize("m,exchange", [(2, 0), (4, 1)])
def test_multi_mode_sharded_device_input(samedev, m, exchange):
    import torch
    import paper_conf_ipps_junger0s18_b200 as wd
    import wdgen.gpu as gg
    n_local = 1 << 20
    n = n_local * m
    with wd.Table(int(math.ceil(n / 0.95)), m, 16, exchange=exchange) as t:
        keys = [gg.unique_keys(n_local, KS, start=r * n_local) for r in range(m)]
        vals = [gg.values(n_local, VS, start=r * n_local) for r in range(m)]
        q = [gg.interleaved_queries(n, KS, start=2 * r * n_local, count=2 * n_local) for r in range(m)]
        vo = [torch.empty(2 * n_local, dtype=torch.int32, device="cuda") for _ in range(m)]
        fo = [torch.empty(2 * n_local, dtype=torch.uint8, device="cuda") for _ in range(m)]
        st = [torch.cuda.Stream() for _ in range(m)]
        with pytest.raises(Exception):
            t.insert(keys[0], vals[0])                     # whole-table call: host memory only
        t.insert_sharded(keys, vals, st)
        t.retrieve_sharded(q, vo, fo, st)
        torch.cuda.synchronize()
        assert t.sync() == 0 and t.size() == n
        for r in range(m):
            bad, first, found = gg.check_unique(q[r], vo[r], fo[r], n, KS, VS)
            assert bad == 0 and found == n_local, (r, bad, first, found)


def test_multi_mode_needs_the_hook(monkeypatch):
    # without the hook a table over more devices than visible is refused
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    import paper_conf_ipps_junger0s18_b200 as wd
    monkeypatch.delenv("WD_MULTI_SAME_DEVICE", raising=False)
    with pytest.raises(Exception):
        wd.Table(1000, torch.cuda.device_count() + 1, 4)
