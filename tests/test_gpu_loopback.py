"""Multi-shard cascade on ONE GPU: m virtual shards (wd_create_loopback) run the full
multi-GPU path — multisplit fused with the push into the owners' receive regions,
T row/column via flags, local insert/query, reverse pull + unpermute — with peer pointers
that happen to be local.  Results must equal the oracle bit for bit (the paper's
"transparent scaling", P:7), and every shard must hold exactly its partition."""
import numpy as np
import pytest

import oracle
import wdgen
from wdtest import capacity_for, from_dev, gpu_roundtrip, to_dev

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def wd():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    import paper_conf_ipps_junger0s18_b200 as wd
    return wd


@pytest.mark.parametrize("m", [2, 3, 4, 8])
@pytest.mark.parametrize("G,mode", [(1, 1), (4, 1), (32, 1), (4, 2), (4, 0)])
def test_loopback_unique_parity(wd, m, G, mode):
    n = 200_000 + 17 * m
    keys, vals = wdgen.unique_keys(n, 21), wdgen.values(n, 22)
    q = wdgen.interleaved_queries(n, 21)
    with wd.Table(capacity_for(n, 0.9), group_size=G, loopback_shards=m) as t:
        t.set_option(wd.WD_OPT_PROBE_MODE, mode)
        t.set_option(wd.WD_OPT_QUERY_GROUP_SIZE, -1 if mode == 0 else 0)   # 0: the table's |g|
        t.set_option(wd.WD_OPT_INSERT_GROUP_SIZE, -1 if mode == 0 else 0)
        t.set_option(wd.WD_OPT_BATCH, 9_000)  # many batches per shard: epochs wrap slots
        gv, gf = gpu_roundtrip(t, keys, vals, q)
        assert t.sync() == 0, wd._lib.wd_last_error_message()
        assert t.size() == n
        seed = t.get_option(wd.WD_OPT_PART_SEED)
        # shard d holds exactly the keys with p(k) = d
        for d in range(m):
            sl = t.dump(d)
            k = (sl & np.uint64(0xFFFFFFFF)).astype(np.uint32)
            k = k[k != np.uint32(0xFFFFFFFF)]
            assert np.all(oracle.partition(k, m, seed) == d)
            assert t.counters(d)["exchange_errors"] == 0
    cv, cf = oracle.expected_unique(q, n, 21, 22)
    assert np.array_equal(gf, cf) and np.array_equal(gv, cv)


@pytest.mark.parametrize("m", [2, 4])
def test_loopback_host_and_dups(wd, m):
    n = 120_000
    keys = wdgen.uniform_keys(n, 31) % np.uint32(50_000)
    vals = wdgen.values(n, 32)
    q = np.arange(60_000, dtype=np.uint32)
    with wd.Table(capacity_for(50_000, 0.85), group_size=4, loopback_shards=m) as t:
        t.set_option(wd.WD_OPT_BATCH, 5_000)
        gv, gf = gpu_roundtrip(t, keys, vals, q, host=True)
        assert t.sync() == 0
        mo = oracle.Map(n, dup_mode=True)
        mo.insert(keys, vals)
        assert t.size() == mo.size()
    ev, ef = mo.retrieve(q)
    assert np.array_equal(gf, ef)
    assert np.all(mo.pair_status(q[gf == 1], gv[gf == 1]) >= 1)


def test_loopback_fig4_partition_mode(wd):
    # Fig. 4: p(k) = k mod 4 over 4 shards
    keys = np.arange(1, 4001, dtype=np.uint32) * 3
    vals = keys ^ np.uint32(0xABCDEF)
    with wd.Table(6000, group_size=2, loopback_shards=4) as t:
        t.set_option(wd.WD_OPT_PART_MODE, 1)
        t.set_option(wd.WD_OPT_BATCH, 333)
        gv, gf = gpu_roundtrip(t, keys, vals, np.concatenate([keys, keys + 1]))
        for d in range(4):
            sl = t.dump(d)
            k = (sl & np.uint64(0xFFFFFFFF)).astype(np.uint32)
            k = k[k != np.uint32(0xFFFFFFFF)]
            assert np.all(k % 4 == d)
        assert t.size() == keys.size
    assert np.all(gf[:4000] == 1) and np.array_equal(gv[:4000], vals)
    kk = keys + 1
    present = np.isin(kk, keys)
    assert np.array_equal(gf[4000:].astype(bool), present)


def test_loopback_uneven_and_empty(wd):
    # one call with fewer items than shards, then n = 0
    with wd.Table(1000, group_size=4, loopback_shards=8) as t:
        gv, gf = gpu_roundtrip(t, np.array([5, 6, 7], np.uint32), np.array([1, 2, 3], np.uint32),
                               np.array([7, 6, 5, 4], np.uint32))
        assert list(gf) == [1, 1, 1, 0] and list(gv[:3]) == [3, 2, 1]
        t.insert(to_dev(np.zeros(0, np.uint32)), to_dev(np.zeros(0, np.uint32)))
        assert t.sync() == 0 and t.size() == 3


@pytest.mark.parametrize("m", [2, 8])
def test_loopback_zipf(wd, m):
    # partition skew of Zipf inputs: the hottest keys all land on one shard
    n = 1 << 19
    keys = wdgen.zipf_keys(n, 2**32 - 1, 27)
    vals = wdgen.values(n, 28)
    distinct = np.unique(keys).size
    with wd.Table(capacity_for(distinct, 0.9), group_size=4, loopback_shards=m, batch=30_000) as t:
        q = np.unique(keys)
        gv, gf = gpu_roundtrip(t, keys, vals, q)
        assert t.sync() == 0
        assert t.size() == distinct
    mo = oracle.Map(n, dup_mode=True)
    mo.insert(keys, vals)
    assert np.all(gf == 1)
    assert np.all(mo.pair_status(q, gv) >= 1)


@pytest.mark.parametrize("m", [2, 4])
def test_loopback_sharded_calls(wd, m):
    # wd_insert_sharded / wd_retrieve_sharded (the device-sided cascade of
    # P:175 / P:199): every shard brings its own device-resident portion on its own stream;
    # every query of every portion against the closed form
    import torch
    import wdgen.gpu as gg
    n_local, ks, vs = 150_001, 91, 92
    n = n_local * m
    with wd.Table(capacity_for(n, 0.9), group_size=8, loopback_shards=m) as t:
        t.set_option(wd.WD_OPT_BATCH, 40_000)
        assert t.get_option(wd.WD_OPT_LOCAL_SHARDS) == m
        keys = [gg.unique_keys(n_local, ks, start=r * n_local) for r in range(m)]
        vals = [gg.values(n_local, vs, start=r * n_local) for r in range(m)]
        streams = [torch.cuda.Stream() for _ in range(m)]
        for s in streams:                        # the portions were generated on this stream
            s.wait_stream(torch.cuda.current_stream())
        t.insert_sharded(keys, vals, streams)
        q = [gg.interleaved_queries(n, ks, start=r * 2 * n_local, count=2 * n_local) for r in range(m)]
        vo = [torch.empty(2 * n_local, dtype=torch.int32, device="cuda") for _ in range(m)]
        fo = [torch.empty(2 * n_local, dtype=torch.uint8, device="cuda") for _ in range(m)]
        for s in streams:
            s.wait_stream(torch.cuda.current_stream())
        t.retrieve_sharded(q, vo, fo, streams)
        torch.cuda.synchronize()
        assert t.sync() == 0 and t.size() == n
        for r in range(m):
            bad, first, found = gg.check_unique(q[r], vo[r], fo[r], n, ks, vs)
            assert bad == 0, (r, bad, first)
            assert found == n_local
        with pytest.raises(ValueError):
            t.insert_sharded(keys[:1], vals[:1])


@pytest.mark.parametrize("m", [2, 3, 8])
@pytest.mark.parametrize("exchange", [0, 1])
def test_loopback_exchange_modes(wd, m, exchange):
    # WD_OPT_EXCHANGE: fused peer stores (0) and the staged copy-engine transposition (1,
    # the paper's asynchronous inter-GPU copies) must give identical maps: unique keys over
    # many batches (epochs wrap both exchange slots), host and device buffers, duplicates,
    # erase through the reverse path
    import torch
    n = 250_007
    keys, vals = wdgen.unique_keys(n, 81), wdgen.values(n, 82)
    q = wdgen.interleaved_queries(n, 81)
    with wd.Table(capacity_for(n, 0.9), group_size=8, loopback_shards=m, exchange=exchange) as t:
        assert t.get_option(wd.WD_OPT_EXCHANGE) == exchange
        t.set_option(wd.WD_OPT_BATCH, 20_000)
        gv, gf = gpu_roundtrip(t, keys, vals, q)
        assert t.sync() == 0 and t.size() == n
        hv, hf = gpu_roundtrip(t, keys[:0], vals[:0], q, host=True)
        er = t.erase(to_dev(q[: n // 2]))
        torch.cuda.synchronize()
        assert t.sync() == 0
    cv, cf = oracle.expected_unique(q, n, 81, 82)
    assert np.array_equal(gf, cf) and np.array_equal(gv, cv)
    assert np.array_equal(hf, cf) and np.array_equal(hv, cv)
    assert np.array_equal(er.cpu().numpy().astype(bool), cf[: n // 2].astype(bool))
    dk = wdgen.uniform_keys(300_000, 83) % np.uint32(70_000)
    dv = wdgen.values(300_000, 84)
    with wd.Table(capacity_for(70_000, 0.9), group_size=4, loopback_shards=m, exchange=exchange) as t:
        t.set_option(wd.WD_OPT_BATCH, 30_000)
        qq = np.arange(71_000, dtype=np.uint32)
        gv, gf = gpu_roundtrip(t, dk, dv, qq)
        mo = oracle.Map(300_000, dup_mode=True)
        mo.insert(dk, dv)
        assert t.sync() == 0 and t.size() == mo.size()
    ev, ef = mo.retrieve(qq)
    assert np.array_equal(gf, ef)
    assert np.all(mo.pair_status(qq[gf == 1], gv[gf == 1]) >= 1)


def test_loopback_rejects_nccl_exchange(wd):
    with wd.Table(1000, group_size=4, loopback_shards=2) as t:
        with pytest.raises(wd.WarpDriveError) as ei:
            t.set_option(wd.WD_OPT_EXCHANGE, 2)
        assert ei.value.status == wd.WD_ERR_UNSUPPORTED
        with pytest.raises(wd.WarpDriveError):
            t.set_option(wd.WD_OPT_EXCHANGE, 3)


def test_phase_times_decomposition(wd):
    # wd_phase_times (Fig. 11 decomposition): the phases each path runs are reported, with
    # positive times; off by default; reading resets
    import torch
    import wdgen.gpu as gg
    n = 1 << 22
    keys, vals = gg.unique_keys(n, 301), gg.values(n, 302)
    with wd.Table(capacity_for(n, 0.9), group_size=8, loopback_shards=2, batch=1 << 20,
                  exchange=1) as t:
        t.insert(keys, vals)
        assert all(c == 0 for _, c in t.phase_times().values())      # off: nothing recorded
        t.set_option(wd.WD_OPT_PHASE_TIMING, 1)
        t.insert(keys, vals)
        ph = t.phase_times()
        assert {k for k, (ms, c) in ph.items() if c} == {"multisplit", "exchange", "probe"}
        assert all(ms > 0 for ms, c in ph.values() if c)
        vo = torch.empty(n, dtype=torch.int32, device="cuda")
        fo = torch.empty(n, dtype=torch.uint8, device="cuda")
        t.retrieve(keys, vo, fo)
        ph = t.phase_times()
        assert {k for k, (ms, c) in ph.items() if c} == {"multisplit", "exchange", "probe_query",
                                                          "reverse", "unpermute"}
        assert gg.check_unique(keys, vo, fo, n, 301, 302)[0] == 0
    with wd.Table(capacity_for(n, 0.9), 1, 16) as t:
        t.set_option(wd.WD_OPT_PHASE_TIMING, 1)
        t.set_option(wd.WD_OPT_SLICES, 4)
        t.insert(keys, vals)
        assert {k for k, (ms, c) in t.phase_times().items() if c} == {"group", "probe"}
        hk = keys.cpu().pin_memory()
        t.retrieve(hk)
        assert {k for k, (ms, c) in t.phase_times().items() if c} == {"h2d", "probe_query", "d2h"}


def test_sharded_host_portions(wd):
    # _sharded calls with pinned host portions: streamed per shard (a11) through the cascade
    import torch
    n_local, m = 70_001, 3
    n = n_local * m
    with wd.Table(capacity_for(n, 0.9), group_size=4, loopback_shards=m, batch=20_000) as t:
        ks = [torch.from_numpy(wdgen.unique_keys(n_local, 311, start=r * n_local).view(np.int32)).pin_memory()
              for r in range(m)]
        vs = [torch.from_numpy(wdgen.values(n_local, 312, start=r * n_local).view(np.int32)).pin_memory()
              for r in range(m)]
        t.insert_sharded(ks, vs)
        vo = [torch.empty(n_local, dtype=torch.int32).pin_memory() for _ in range(m)]
        fo = [torch.empty(n_local, dtype=torch.uint8).pin_memory() for _ in range(m)]
        t.retrieve_sharded(ks, vo, fo)
        torch.cuda.synchronize()
        assert t.sync() == 0 and t.size() == n
    for r in range(m):
        cv, cf = oracle.expected_unique(ks[r].numpy().view(np.uint32), n, 311, 312)
        assert np.array_equal(fo[r].numpy(), cf) and np.array_equal(vo[r].numpy().view(np.uint32), cv)
